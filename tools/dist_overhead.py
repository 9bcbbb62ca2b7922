"""Per-round overhead of the balanced multi-GPU protocol: virtual ranks on a tiny spec (kernel work
~0), serialized; and the single-GPU per-round cost on the same spec.   python tools/dist_overhead.py"""
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

out = {}
for R in (64, 512):
    spec = A.c5_chains(R, 8)
    res = {}
    for N in (1, 2, 8):
        spaces = [Space(spec, flags=L.ATF_FLAG_NO_SEG_BOUNDS) for _ in range(N)]
        virtual_ranks(spaces)
        best = None
        for _ in range(5):
            vag = virtual_ranks(spaces, serialize=True)
            rr = [round(max(vag.round_s[r][i] for r in range(N)) * 1e3, 3) for i in range(len(vag.round_s[0]))]
            if best is None or sum(rr) < sum(best):
                best = rr
        res[N] = best
        for sp in spaces:
            sp.close()
    with Space(spec, flags=L.ATF_FLAG_NO_SEG_BOUNDS) as sp:
        sp.generate()
        ts = []
        for fl in (0, 1):
            pass
        for _ in range(10):
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            sp.generate()
            torch.cuda.synchronize()
            ts.append((time.perf_counter() - t0) * 1e3)
        res["single_generate_ms_replay"] = min(ts)
    with Space(spec, flags=L.ATF_FLAG_NO_SEG_BOUNDS | L.ATF_FLAG_NO_REPLAY) as sp:
        sp.generate()
        ts = []
        for _ in range(10):
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            sp.generate()
            torch.cuda.synchronize()
            ts.append((time.perf_counter() - t0) * 1e3)
        res["single_generate_ms_per_level_sync"] = min(ts)
    out[f"C5-{R}x8"] = res
print(json.dumps(out))
