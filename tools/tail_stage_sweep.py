"""Tail emit staging size per warp vs C3-IS2 / IS4 generation time (atf_test_set_tail_stage):
python tools/tail_stage_sweep.py [bytes ...]"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import atfspec as A  # noqa: E402
from paper_conf_hpdc_raschg18_b200 import Space, _lib as L  # noqa: E402

stages = [int(x) for x in sys.argv[1:]] or [4096, 6144, 8192, 12288]
flush = torch.empty(128 << 20, dtype=torch.int32, device="cuda")
out = {}
for st in stages:
    L.check(L.atf_test_set_tail_stage(st))
    for name in ("IS2", "IS4"):
        with Space(A.c3_xgemm(name), flags=L.ATF_FLAG_NO_SEG_BOUNDS) as sp:
            for _ in range(3):
                sp.generate()
            ts = []
            for _ in range(10):
                flush.add_(1)
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record()
                sp.generate()
                e1.record()
                torch.cuda.synchronize()
                ts.append(e0.elapsed_time(e1))
            out[f"{name}@{st}"] = round(sorted(ts)[len(ts) // 2], 4)
            print(name, st, out[f"{name}@{st}"], flush=True)
L.check(L.atf_test_set_tail_stage(0))
print(json.dumps(out))
