#!/bin/bash
# quick GPU check: parity subset (-k $K), C3 launch lists, bench.  T=tag K=pytest-k-expr
mkdir -p gpurun_out
T=${T:-quick}
K=${K:-"tail or C3 or golden or fuzz"}
timeout 1200 python -m pytest tests -m gpu -q -x -k "$K" > gpurun_out/${T}_pytest_gpu.txt 2>&1
echo "pytest rc=$?" >> gpurun_out/${T}_pytest_gpu.txt
tail -2 gpurun_out/${T}_pytest_gpu.txt
for cfg in ${CFGS:-C3-IS4 C3-IS2}; do
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${T}_launches_${cfg}.csv python tools/gen_once.py $cfg --reps 2 --profile-last > /dev/null 2>&1
  echo "launches $cfg rc=$?"
done
if [ -n "$NCU" ]; then
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:$NCU -c ${NCUC:-4} -o gpurun_out/${T}_ncu python tools/gen_once.py ${NCUCFG:-C3-IS2} > /dev/null 2>&1; echo "ncu rc=$?"
fi
if [ -z "$NOBENCH" ]; then
  timeout 1200 python bench.py --steps 10 > gpurun_out/${T}_bench.json 2> gpurun_out/${T}_bench.err; echo "bench rc=$?"
  python tools/bench_brief.py gpurun_out/${T}_bench.json 2>/dev/null | head -20
fi
