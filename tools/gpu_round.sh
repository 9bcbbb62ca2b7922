#!/bin/bash
# One gpurun round trip: GPU tests, a short bench, an ncu launch list of one C5 generation.
# usage (under gpurun): bash tools/gpu_round.sh TAG [bench-args...]
TAG=${1:-x}; shift
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/${TAG}_gpu.txt 2>&1
timeout 900 python -m pytest tests -m gpu -q --maxfail=5 > gpurun_out/${TAG}_pytest_gpu.txt 2>&1
echo "pytest rc=$?" >> gpurun_out/${TAG}_pytest_gpu.txt
tail -3 gpurun_out/${TAG}_pytest_gpu.txt
if [ -n "$BENCH" ]; then
  timeout 900 python bench.py $BENCH > gpurun_out/${TAG}_bench.json 2> gpurun_out/${TAG}_bench.err
  echo "bench rc=$?"; tail -c 3000 gpurun_out/${TAG}_bench.json
fi
if [ -n "$LAUNCHES" ]; then
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
    --log-file gpurun_out/${TAG}_launches.csv python tools/gen_once.py $LAUNCHES > /dev/null 2>&1
  echo "ncu launches rc=$?"
fi
