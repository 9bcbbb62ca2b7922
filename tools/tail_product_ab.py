"""A/B of the product-structured fused tail vs the depth-first tail kernels (atf_test_set_tail_product):
medians of 10 steady-state generations (L2 flushed) of C3-IS2 / IS4 / C2.   python tools/tail_product_ab.py"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

import atfspec as A  # noqa: E402
from paper_conf_hpdc_raschg18_b200 import Space, _lib as L  # noqa: E402

flush = torch.empty(128 << 20, dtype=torch.int32, device="cuda")
for rep in range(2):
    for on in (1, 0):
        L.check(L.atf_test_set_tail_product(on))
        out = []
        for name in ("C3-IS2", "C3-IS4", "C2"):
            with Space(A.config_spec(name)) as sp:
                for _ in range(3):
                    sp.generate()
                ts = []
                for _ in range(10):
                    flush.add_(1)
                    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                    a.record()
                    sp.generate()
                    b.record()
                    torch.cuda.synchronize()
                    ts.append(a.elapsed_time(b))
                out.append(f"{name} {np.median(ts):.3f}")
            with Space(A.config_spec(name), flags=L.ATF_FLAG_TIMING | L.ATF_FLAG_SERIAL_GROUPS) as sp:
                for _ in range(2):
                    sp.generate()
                tail = [round(s["ms"], 4) for s in sp.stats() if s["kernel"] in (5, 6) and s["ms"] > 0]
                out.append(f"tail {tail}")
        print("product" if on else "dfs    ", " ".join(out), flush=True)
L.check(L.atf_test_set_tail_product(1))
