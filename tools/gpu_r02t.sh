#!/bin/bash
mkdir -p gpurun_out
T=r02t
timeout 900 python -m pytest tests -m gpu -q -x -k "dist" > gpurun_out/${T}_pytest_gpu.txt 2>&1; echo "pytest rc=$?" >> gpurun_out/${T}_pytest_gpu.txt
tail -2 gpurun_out/${T}_pytest_gpu.txt
for N in 1 8; do
  timeout 900 ncu --profile-from-start off --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${T}_dist_launches_N$N.csv python tools/dist_launches.py $N > /dev/null 2>&1; echo "dist launches N=$N rc=$?"
done
