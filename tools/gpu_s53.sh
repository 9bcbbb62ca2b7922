mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q -x > gpurun_out/s53_pytest.txt 2>&1; echo pytest rc=$?; tail -3 gpurun_out/s53_pytest.txt
timeout 600 ncu --set full --clock-control none --import-source on -k regex:expand_wtile --launch-skip 21 --launch-count 3 -o gpurun_out/r01s53_c5_l8 python tools/gen_once.py C5 > gpurun_out/s53_ncu.log 2>&1; echo ncu rc=$?
python tools/traffic_db.py gpurun_out/r01s53_c5_l8.ncu-rep C5_chains_4096x8:g0:l7,C5_chains_4096x8:g1:l7,C5_chains_4096x8:g2:l7 > /dev/null 2>&1; cp profiles/traffic.json gpurun_out/traffic.json
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/s53_launches.csv python tools/gen_once.py C5 > /dev/null 2>&1; echo launches rc=$?
timeout 900 python bench.py > gpurun_out/s53_bench.json 2> gpurun_out/s53_bench.err; echo bench rc=$?
cat gpurun_out/s53_bench.json
timeout 200 python tools/level_frac.py C5 5 > gpurun_out/s53_lf_C5.txt 2>&1
timeout 200 python tools/level_frac.py C3-IS2 5 > gpurun_out/s53_lf_C3.txt 2>&1
