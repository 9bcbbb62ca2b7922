"""Per-level sizes of a config under several flag sets vs the oracle (debug aid):
python tools/debug_levels.py C3-IS1"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import atfspec as A  # noqa: E402
from oracle import run as orc  # noqa: E402
from paper_conf_hpdc_raschg18_b200 import Space, _lib as L  # noqa: E402

spec = A.config_spec(sys.argv[1]) if sys.argv[1] in A.CONFIGS else eval(sys.argv[1])
ref = orc.info(spec, threads=8)
print("oracle", [[lv["f"] for lv in g["levels"]] for g in ref["groups"]])
base = None
for name, fl in [("default", 0), ("no_jit", L.ATF_FLAG_NO_JIT), ("no_tail", L.ATF_FLAG_NO_TAIL),
                 ("no_jit_no_tail", L.ATF_FLAG_NO_JIT | L.ATF_FLAG_NO_TAIL)]:
    with Space(spec, flags=fl | L.ATF_FLAG_TIMING) as sp:
        sp.generate()
        print(name, [sp.level_sizes(g) for g in range(sp.num_groups())],
              [st["kernel"] for st in sp.stats() if st["group"] == 0])
        recs = [sp.level_tensors(0, k)[0].cpu() for k in range(sp.num_levels(0))]
        if base is None:
            base = recs
        else:
            for k, (a, b) in enumerate(zip(base, recs)):
                if a.shape != b.shape or not a.equal(b):
                    print("   level", k, "differs from default")
