#!/bin/bash
mkdir -p gpurun_out
T=${T:-r02i}
timeout 2400 python -m pytest tests -m gpu -q --maxfail=5 --durations=20 > gpurun_out/${T}_pytest_gpu.txt 2>&1
echo "pytest rc=$?" >> gpurun_out/${T}_pytest_gpu.txt
tail -3 gpurun_out/${T}_pytest_gpu.txt
timeout 600 ncu --set full --clock-control none --import-source on -k regex:decode -c 1 -o gpurun_out/${T}_decode_c4 python tools/gen_once.py C3-IS2 --decode 100000000 > gpurun_out/${T}_ncu_decode.log 2>&1
echo "ncu decode rc=$?"
timeout 1200 python bench.py --steps 10 > gpurun_out/${T}_bench.json 2> gpurun_out/${T}_bench.err; echo "bench rc=$?"
python tools/bench_brief.py gpurun_out/${T}_bench.json 2>/dev/null | head -20
timeout 1500 python tools/cpu_baselines.py > gpurun_out/${T}_cpu_baselines.json 2> gpurun_out/${T}_cpu_baselines.err; echo "cpu baselines rc=$?"
