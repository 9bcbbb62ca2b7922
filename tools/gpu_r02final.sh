#!/bin/bash
# round-2 final GPU evidence: every GPU test, smoke, sanitizers, launch lists, ncu --set full of
# the dominant C5 launch and of C3-IS2's tail, bench
mkdir -p gpurun_out
T=${T:-r02x}
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/${T}_gpu.txt 2>&1
timeout 2400 python -m pytest tests -m gpu -q --maxfail=10 --durations=15 > gpurun_out/${T}_pytest_gpu.txt 2>&1
echo "pytest rc=$?" >> gpurun_out/${T}_pytest_gpu.txt; tail -3 gpurun_out/${T}_pytest_gpu.txt
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${T}_smoke.txt 2>&1; echo "smoke rc=$?"
for tool in ${SANITIZE:-}; do
  timeout 1500 compute-sanitizer --tool $tool --print-limit 50 python tools/sanitize_run.py > gpurun_out/${T}_sanitize_$tool.txt 2>&1
  echo "sanitize $tool rc=$?"; tail -2 gpurun_out/${T}_sanitize_$tool.txt
done
for cfg in C5 C3-IS2 C3-IS4; do
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${T}_launches_${cfg}.csv python tools/gen_once.py $cfg --reps 2 --profile-last > /dev/null 2>&1
  echo "launches $cfg rc=$?"
done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:expand_wtile --launch-skip 21 --launch-count 2 -o gpurun_out/${T}_c5_l8 python tools/gen_once.py C5 > /dev/null 2>&1; echo "ncu c5 l8 rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:atf_tail -c 2 -o gpurun_out/${T}_tail_is2 python tools/gen_once.py C3-IS2 > /dev/null 2>&1; echo "ncu tail is2 rc=$?"
timeout 1200 python bench.py --steps 10 > gpurun_out/${T}_bench.json 2> gpurun_out/${T}_bench.err; echo "bench rc=$?"
python tools/bench_brief.py gpurun_out/${T}_bench.json 2>/dev/null | head -24
