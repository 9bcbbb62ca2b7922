#!/bin/bash
# A/B timing of one build under different environments (medians of 10 warm generations).
# usage (under gpurun): bash tools/ab_env.sh "" "VAR=1" ...
for i in 1 2; do
for E in "$@"; do
env $E python - "$E" <<'PY'
import sys, torch, numpy as np, atfspec as A
from paper_conf_hpdc_raschg18_b200 import Space
out = []
for name, spec in (("C5", A.c5_chains(4096, 8)), ("C3-IS2", A.c3_xgemm("IS2")), ("C2", A.c2_xgemm_direct(256))):
    with Space(spec) as sp:
        for _ in range(3): sp.generate()
        torch.cuda.synchronize(); ts = []
        for _ in range(10):
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(); sp.generate(); b.record(); torch.cuda.synchronize(); ts.append(a.elapsed_time(b))
        out.append(f"{name} {np.median(ts):.3f}")
print(f"[{sys.argv[1]}]", " ".join(out), flush=True)
PY
done; done
