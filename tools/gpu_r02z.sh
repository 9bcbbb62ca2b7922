#!/bin/bash
# re-entry check of HEAD: every GPU test, smoke, bench, C5 / C3 launch lists
mkdir -p gpurun_out
T=${T:-r02z}
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/${T}_gpu.txt 2>&1
timeout 2400 python -m pytest tests -m gpu -q --maxfail=10 --durations=25 > gpurun_out/${T}_pytest_gpu.txt 2>&1
echo "pytest rc=$?" >> gpurun_out/${T}_pytest_gpu.txt
tail -3 gpurun_out/${T}_pytest_gpu.txt
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${T}_smoke.txt 2>&1; echo "smoke rc=$?"
timeout 1200 python bench.py --steps 10 > gpurun_out/${T}_bench.json 2> gpurun_out/${T}_bench.err; echo "bench rc=$?"
python tools/bench_brief.py gpurun_out/${T}_bench.json 2>/dev/null | head -24
for cfg in C5 C3-IS2; do
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${T}_launches_${cfg}.csv python tools/gen_once.py $cfg --reps 2 --profile-last > /dev/null 2>&1
  echo "launches $cfg rc=$?"
done
