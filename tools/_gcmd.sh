mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q -x --maxfail=3 > gpurun_out/r01s5_pytest.txt 2>&1; echo "pytest rc=$?"; tail -15 gpurun_out/r01s5_pytest.txt
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r01s5_launches.csv python tools/gen_once.py C5 > /dev/null 2>&1; echo "ncu rc=$?"
timeout 600 python bench.py --steps 10 --warmup 3 --no-secondary --cpu-budget 2 > gpurun_out/r01s5_bench.json 2> gpurun_out/r01s5_bench.err; echo "bench rc=$?"; tail -c 1500 gpurun_out/r01s5_bench.json; tail -5 gpurun_out/r01s5_bench.err
