#!/bin/bash
# A/B timing of the current tree vs the package copy in build/ab_old_tree (its own binding and
# libatfgen.so), medians of 10 warm generations, headline flags for C5.  usage (under gpurun)
for i in 1 2; do
for D in "$PWD" "$PWD/build/ab_old_tree"; do
(cd "$D" && python - "$D" <<'PY'
import sys, os
sys.path.insert(0, os.getcwd())
import torch, numpy as np, atfspec as A
from paper_conf_hpdc_raschg18_b200 import Space, _lib as L
out = []
for name, spec, fl in (("C5", A.c5_chains(4096, 8), L.ATF_FLAG_NO_SEG_BOUNDS), ("C3-IS2", A.c3_xgemm("IS2"), 0),
                       ("C3-IS4", A.c3_xgemm("IS4"), 0), ("C2", A.c2_xgemm_direct(256), 0)):
    with Space(spec, flags=fl) as sp:
        for _ in range(3): sp.generate()
        torch.cuda.synchronize(); ts = []
        for _ in range(10):
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(); sp.generate(); b.record(); torch.cuda.synchronize(); ts.append(a.elapsed_time(b))
        out.append(f"{name} {np.median(ts):.3f}")
print(sys.argv[1].split("/")[-1], " ".join(out), flush=True)
PY
)
done; done
