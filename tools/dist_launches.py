"""Kernel launches of a balanced generation over N virtual ranks (for an ncu launch list):
serialized virtual ranks (one rank's round at a time on the GPU); the third generation is
bracketed by cudaProfilerStart/Stop.   ncu --profile-from-start off ... python tools/dist_launches.py N"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import atfspec as A  # noqa: E402
from paper_conf_hpdc_raschg18_b200 import Space, _lib as L  # noqa: E402
from paper_conf_hpdc_raschg18_b200.shard import VirtualAllGather  # noqa: E402
import threading  # noqa: E402

N = int(sys.argv[1]) if len(sys.argv) > 1 else 8
R = int(sys.argv[2]) if len(sys.argv) > 2 else 0
spec = A.c5_chains(4096, 8)
spaces = [Space(spec, flags=L.ATF_FLAG_NO_SEG_BOUNDS | L.ATF_FLAG_NO_REPLAY) for _ in range(N)]


def gen(profile):
    vag = VirtualAllGather(N, serialize=True)
    errs = []

    def run(r):
        try:
            torch.cuda.set_device(0)
            vag.start(r)
            spaces[r].generate_dist(r, N, lambda b: vag(r, b))
            torch.cuda.synchronize()
            vag.finish(r)
        except Exception as ex:  # noqa: BLE001
            errs.append(ex)
            vag.barrier.abort()
    th = [threading.Thread(target=run, args=(r,)) for r in range(N)]
    for t in th:
        t.start()
    for t in th:
        t.join()
    if errs:
        raise errs[0]


gen(False)
gen(False)
torch.cuda.synchronize()
torch.cuda.cudart().cudaProfilerStart()
gen(True)
torch.cuda.synchronize()
torch.cuda.cudart().cudaProfilerStop()
print("ok")
