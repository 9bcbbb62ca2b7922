"""C5 / C3-IS2 / C2 generation time (one GPU, steady state, L2 flushed) and the one-GPU 8-rank
prediction (sync protocol) vs the in-place threshold of warp-tile levels (atf_test_set_direct_tiles):
python tools/direct_sweep.py 16 64 256 ..."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import atfspec as A  # noqa: E402
from paper_conf_hpdc_raschg18_b200 import Space, _lib as L  # noqa: E402
from paper_conf_hpdc_raschg18_b200.shard import virtual_ranks  # noqa: E402

flush = torch.empty(128 << 20, dtype=torch.int32, device="cuda")


def one_gpu(spec, flags):
    with Space(spec, flags=flags) as sp:
        for _ in range(3):
            sp.generate()
        ts = []
        for _ in range(8):
            flush.add_(1)
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            sp.generate()
            e1.record()
            torch.cuda.synchronize()
            ts.append(e0.elapsed_time(e1))
    return round(sorted(ts)[len(ts) // 2], 3)


out = {}
c5 = A.c5_chains(4096, 8)
for arg in sys.argv[1:]:
    L.check(L.atf_test_set_direct_tiles(int(arg)))
    res = {"c5_ms": one_gpu(c5, L.ATF_FLAG_NO_SEG_BOUNDS), "c3is2_ms": one_gpu(A.c3_xgemm("IS2"), 0),
           "c2_ms": one_gpu(A.c2_xgemm_direct(256), 0)}
    for N in (1, 8):
        spaces = [Space(c5, flags=L.ATF_FLAG_NO_SEG_BOUNDS | L.ATF_FLAG_NO_REPLAY) for _ in range(N)]
        virtual_ranks(spaces)
        best = None
        for _ in range(3):
            vag = virtual_ranks(spaces, serialize=True)
            rounds = len(vag.round_s[0])
            t = sum(max(vag.round_s[r][i] for r in range(N)) for i in range(rounds)) + (rounds - 1) * 25e-6
            best = t if best is None else min(best, t)
        for sp in spaces:
            sp.close()
        res[f"T{N}_ms"] = round(best * 1e3, 3)
    res["eff8"] = round(res["T1_ms"] / (8 * res["T8_ms"]), 3)
    out[arg] = res
    print(arg, res, flush=True)
L.check(L.atf_test_set_direct_tiles(0))
print(json.dumps(out))
