"""Time the C4 decode (10^8 splitmix64 indices into C3-IS2) alone: python tools/bench_decode.py"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

import atfspec as A  # noqa: E402
from atfspec.fuzz import splitmix64_indices  # noqa: E402
from paper_conf_hpdc_raschg18_b200 import Space  # noqa: E402

spec = A.c3_xgemm("IS2")
with Space(spec) as sp:
    sp.generate()
    S, n = sp.size(), 100_000_000
    idx = torch.from_numpy(splitmix64_indices(n, S, A.c4_indices_seed()).view(np.int64)).cuda()
    out = torch.empty((len(spec.params), n), dtype=torch.int32, device="cuda")
    fl = torch.empty(128 << 20, dtype=torch.int32, device="cuda")
    for _ in range(3):
        sp.decode(idx, out=out)
    ts = []
    for _ in range(5):
        fl.add_(1)
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        sp.decode(idx, out=out)
        b.record()
        torch.cuda.synchronize()
        ts.append(a.elapsed_time(b))
    print("decode ms mean %.3f min %.3f" % (np.mean(ts), np.min(ts)), flush=True)
