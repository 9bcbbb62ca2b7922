"""e2e of C5 through the public API (a fresh space per step, as bench.py's e2e), headline flags:
async per-group rounds on / off (atf_test_set_async_rounds), torch allocator on / off."""
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

import atfspec as A  # noqa: E402
from paper_conf_hpdc_raschg18_b200 import Space, _lib as L  # noqa: E402

spec = A.c5_chains(4096, 8)
for rep in range(2):
    for asyn in (1, 0):
        for ta in (True, False):
            L.check(L.atf_test_set_async_rounds(asyn))
            ts = []
            for i in range(6):
                torch.cuda.synchronize()
                t0 = time.perf_counter()
                with Space(spec, flags=L.ATF_FLAG_NO_SEG_BOUNDS, torch_alloc=ta) as sp:
                    sp.generate()
                    sp.size()
                    sp.group_sizes()
                torch.cuda.synchronize()
                if i:
                    ts.append(time.perf_counter() - t0)
            print(f"async={asyn} torch_alloc={ta}: {1e3 * np.mean(ts):.2f} ms (min {1e3 * min(ts):.2f})", flush=True)
L.check(L.atf_test_set_async_rounds(1))
