#!/bin/bash
mkdir -p gpurun_out
T=${T:-r02l}
timeout 2400 python -m pytest tests -m gpu -q --maxfail=5 --durations=10 > gpurun_out/${T}_pytest_gpu.txt 2>&1
echo "pytest rc=$?" >> gpurun_out/${T}_pytest_gpu.txt
tail -2 gpurun_out/${T}_pytest_gpu.txt
for cfg in C3-IS4 C3-IS2 C5; do
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${T}_launches_${cfg}.csv python tools/gen_once.py $cfg --reps 2 --profile-last > /dev/null 2>&1
  echo "launches $cfg rc=$?"
done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:atf_ -c 8 -o gpurun_out/${T}_jit_is2 python tools/gen_once.py C3-IS2 > /dev/null 2>&1; echo "ncu jit rc=$?"
timeout 600 ncu --set full --clock-control none -k regex:decode -c 1 -o gpurun_out/${T}_decode_c4 python tools/gen_once.py C3-IS2 --decode 100000000 > /dev/null 2>&1; echo "ncu decode rc=$?"
timeout 1200 python bench.py --steps 10 > gpurun_out/${T}_bench.json 2> gpurun_out/${T}_bench.err; echo "bench rc=$?"
python tools/bench_brief.py gpurun_out/${T}_bench.json 2>/dev/null | head -20
