"""bench.py's one-GPU scaling prediction (sync and replay protocols) with the plain partition and
with groups on rank subsets (the default) and with the plain partition (ATF_FLAG_DIST_NO_SUBSETS).""" 
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bench  # noqa: E402
import atfspec as A  # noqa: E402
from paper_conf_hpdc_raschg18_b200 import _lib as L  # noqa: E402

base = bench.headline_flags
spec = A.c5_chains(4096, 8)
out = {}
P = L.ATF_FLAG_DIST_NO_SUBSETS
for name, extra in (("plain", P), ("subsets", 0), ("plain2", P), ("subsets2", 0)):
    bench.headline_flags = lambda extra=extra: base() | extra
    r = bench.predicted_scaling(spec)
    out[name] = {m: {n: (round(v["T_ms"], 3), round(v.get("efficiency", 1.0), 3)) for n, v in r[m].items()} for m in ("sync", "replay")}
    print(name, out[name], flush=True)
print(json.dumps(out))
