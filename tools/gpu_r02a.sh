#!/bin/bash
# round-2 GPU check: tests, sanitizers, bench, launch list
mkdir -p gpurun_out
T=r02a
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/${T}_gpu.txt 2>&1
timeout 1800 python -m pytest tests -m gpu -q --maxfail=10 --durations=25 --deselect "tests/test_gpu_parity.py::test_full_size_against_golden[C5-True]" --deselect "tests/test_gpu_parity.py::test_full_size_against_golden[C5-False]" > gpurun_out/${T}_pytest_gpu.txt 2>&1
echo "pytest rc=$?" >> gpurun_out/${T}_pytest_gpu.txt
tail -3 gpurun_out/${T}_pytest_gpu.txt
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${T}_smoke.txt 2>&1; echo "smoke rc=$?"
timeout 900 python bench.py > gpurun_out/${T}_bench.json 2> gpurun_out/${T}_bench.err; echo "bench rc=$?"
tail -c 1500 gpurun_out/${T}_bench.json
for tool in memcheck racecheck synccheck; do
  timeout 900 compute-sanitizer --tool $tool --print-limit 50 python tools/sanitize_run.py > gpurun_out/${T}_sanitize_$tool.txt 2>&1
  echo "sanitize $tool rc=$?"; tail -2 gpurun_out/${T}_sanitize_$tool.txt
done
