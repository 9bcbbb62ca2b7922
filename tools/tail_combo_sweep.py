"""C3-IS2 / IS4 generation time over (leaf-direct mode, staging bytes) combinations of the fused
tail (atf_test_set_tail_leaf_direct / atf_test_set_tail_stage): medians of 10, L2 flushed."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

import atfspec as A  # noqa: E402
from paper_conf_hpdc_raschg18_b200 import Space, _lib as L  # noqa: E402

flush = torch.empty(128 << 20, dtype=torch.int32, device="cuda")
for mode, stage in ((2, 0), (1, 8192), (1, 10240), (1, 12288), (0, 10240), (1, 16384), (2, 0)):
    L.check(L.atf_test_set_tail_leaf_direct(mode))
    L.check(L.atf_test_set_tail_stage(stage))
    out = []
    for name in ("C3-IS2", "C3-IS4"):
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
    print(f"leaf_direct={mode} stage={stage}", " ".join(out), flush=True)
L.check(L.atf_test_set_tail_leaf_direct(2))
L.check(L.atf_test_set_tail_stage(0))
