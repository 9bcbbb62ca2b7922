"""atf_wide_jit superset group size A/B (atf_test_set_wide_group): identical level arrays with groups
of 4 and 8 on C3-IS1 / C3-IS2 / C2-256 / C3-12x30x8, then medians of 10 steady-state generations (L2
flushed) of C3-IS2 / IS4 / C2 for groups of 8, 16, 4, 2.   python tools/wide_group_ab.py"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

import atfspec as A  # noqa: E402
from paper_conf_hpdc_raschg18_b200 import Space, _lib as L  # noqa: E402


def arrays(spec):
    with Space(spec) as sp:
        sp.generate()
        out = []
        for g in range(sp.num_groups()):
            for k in range(sp.num_levels(g)):
                rec, csr = sp.level_tensors(g, k)
                out.append((rec.cpu().clone() if rec is not None else None, csr.cpu().clone() if csr is not None else None))
        return out


for spec in (A.c3_xgemm("IS1"), A.c3_xgemm("IS2"), A.c2_xgemm_direct(256), A.c3_xgemm((12, 30, 8))):
    res = []
    for on in (4, 8):
        L.check(L.atf_test_set_wide_group(on))
        res.append(arrays(spec))
    same = all((a[0] is None and b[0] is None or torch.equal(a[0], b[0])) and
               (a[1] is None and b[1] is None or torch.equal(a[1], b[1])) for a, b in zip(res[0], res[1]))
    print(spec.name, "identical" if same else "DIFFERENT", flush=True)
    assert same
flush = torch.empty(128 << 20, dtype=torch.int32, device="cuda")
for rep in range(2):
    for on in (8, 16, 4, 2):
        L.check(L.atf_test_set_wide_group(on))
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
        print(f"group {on}", " ".join(out), flush=True)
L.check(L.atf_test_set_wide_group(0))
