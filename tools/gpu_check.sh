#!/bin/bash
# One gpurun round trip: GPU parity tests, an ncu launch list of one C5 generation, a bench.
# usage (under gpurun): TAG=name [BENCHARGS="..."] bash tools/gpu_check.sh
mkdir -p gpurun_out
T=${TAG:-x}
timeout 900 python -m pytest tests -m gpu -q -x --maxfail=3 > gpurun_out/${T}_pytest.txt 2>&1; echo "pytest rc=$?"; tail -4 gpurun_out/${T}_pytest.txt
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${T}_launches.csv python tools/gen_once.py C5 > /dev/null 2>&1; echo "ncu rc=$?"
timeout 900 python bench.py --steps 10 --warmup 3 ${BENCHARGS:---no-secondary --cpu-budget 2} > gpurun_out/${T}_bench.json 2> gpurun_out/${T}_bench.err; echo "bench rc=$?"; tail -3 gpurun_out/${T}_bench.err
