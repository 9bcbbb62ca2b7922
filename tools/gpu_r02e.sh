#!/bin/bash
# after the int64 layout fix: A/B vs the pre-int64 tree, int64 GPU tests, ncu of C5's mid levels
mkdir -p gpurun_out
T=${T:-r02e}
timeout 900 bash tools/ab_tree.sh > gpurun_out/${T}_ab.txt 2>&1; echo "ab rc=$?"; cat gpurun_out/${T}_ab.txt
timeout 600 python -m pytest tests/test_int64_values.py -m gpu -q > gpurun_out/${T}_pytest_i64.txt 2>&1; echo "i64 rc=$?"; tail -2 gpurun_out/${T}_pytest_i64.txt
timeout 900 ncu --set full --clock-control none --import-source on -k regex:expand_wtile --launch-skip 9 --launch-count 5 -o gpurun_out/${T}_c5_mid python tools/gen_once.py C5 > gpurun_out/${T}_ncu.log 2>&1; echo "ncu rc=$?"
