#!/bin/bash
# int64 ranges: their GPU tests, the whole GPU suite, smoke, a bench (C5 regression check)
mkdir -p gpurun_out
T=${T:-r02i64}
timeout 600 python -m pytest tests/test_int64_values.py -m gpu -q -x > gpurun_out/${T}_pytest_i64.txt 2>&1; echo "i64 rc=$?"; tail -15 gpurun_out/${T}_pytest_i64.txt
timeout 2400 python -m pytest tests -m gpu -q --maxfail=10 > gpurun_out/${T}_pytest_gpu.txt 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/${T}_pytest_gpu.txt
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${T}_smoke.txt 2>&1; echo "smoke rc=$?"
timeout 1200 python bench.py --steps 10 > gpurun_out/${T}_bench.json 2> gpurun_out/${T}_bench.err; echo "bench rc=$?"
python tools/bench_brief.py gpurun_out/${T}_bench.json 2>/dev/null | head -12
