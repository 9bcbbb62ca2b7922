#!/bin/bash
# int64 GPU tests, A/B of the int64 change on the hot kernels, dist launch lists (N = 1 and 8)
mkdir -p gpurun_out
T=${T:-r02d}
timeout 600 python -m pytest tests/test_int64_values.py -m gpu -q > gpurun_out/${T}_pytest_i64.txt 2>&1; echo "i64 rc=$?"; tail -3 gpurun_out/${T}_pytest_i64.txt
timeout 900 bash tools/ab_tree.sh > gpurun_out/${T}_ab.txt 2>&1; echo "ab rc=$?"; cat gpurun_out/${T}_ab.txt
for N in 1 8; do
  timeout 900 ncu --profile-from-start off --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${T}_dist${N}.csv python tools/dist_launches.py $N > gpurun_out/${T}_dist${N}.log 2>&1; echo "dist$N rc=$?"
done
