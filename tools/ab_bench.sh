#!/bin/bash
# A/B timing of the current build vs build/ab_old/libatfgen.so on one box (medians of 10
# warm generations per config).  usage (under gpurun): [AB_ENV="VAR=1"] bash tools/ab_bench.sh
for i in 1 2; do
for L in paper_conf_hpdc_raschg18_b200/libatfgen.so build/ab_old/libatfgen.so; do
env $AB_ENV ATF_LIB_PATH=$PWD/$L python - <<'PY'
import os, torch, numpy as np, atfspec as A
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
print(os.environ["ATF_LIB_PATH"].split("/")[-2], " ".join(out), flush=True)
PY
done; done
