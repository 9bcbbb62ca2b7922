"""Where the per-round time of the balanced multi-GPU protocol goes (one GPU, virtual ranks):
per rank and round, host time (serialized ranks) vs the device time of the rank's level kernels
(ATF_FLAG_TIMING events).   python tools/dist_probe.py [N]"""
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import atfspec as A  # noqa: E402
from paper_conf_hpdc_raschg18_b200 import Space, _lib as L  # noqa: E402
from paper_conf_hpdc_raschg18_b200.shard import virtual_ranks  # noqa: E402

N = int(sys.argv[1]) if len(sys.argv) > 1 else 8
spec = A.c5_chains(4096, 8)
out = {}
for timing in (0, L.ATF_FLAG_TIMING):
    spaces = [Space(spec, flags=L.ATF_FLAG_NO_SEG_BOUNDS | timing) for _ in range(N)]
    virtual_ranks(spaces)
    vag = virtual_ranks(spaces, serialize=True)
    rec = {"round_ms": [[round(x * 1e3, 3) for x in vag.round_s[r]] for r in range(N)]}
    if timing:
        lv = []
        for sp in spaces:
            st = sp.stats()
            lv.append([[round(x["ms"], 3) for x in st if x["level"] == k] for k in range(8)])
        rec["level_device_ms"] = lv
    out["timing" if timing else "plain"] = rec
    for sp in spaces:
        sp.close()
# single-GPU reference: plain generate, per-level device times (serialized groups)
with Space(spec, flags=L.ATF_FLAG_NO_SEG_BOUNDS | L.ATF_FLAG_TIMING | L.ATF_FLAG_SERIAL_GROUPS) as sp:
    sp.generate()
    sp.generate()
    st = sp.stats()
    out["single_level_ms"] = [[round(x["ms"], 3) for x in st if x["level"] == k] for k in range(8)]
print(json.dumps(out))
