"""Small generations + decodes for compute-sanitizer (racecheck / synccheck / memcheck).

Covers every kernel family of the generation path on small specs: the warp-tile kernel
with the decoupled look-back of tiny in-place levels and the stash + scan + level_emit path
(C5-300x4, C2-256), the NVRTC-specialised and generic narrow fast kernels (C3-IS1), the
fused narrow tail (C2, C3), decode / encode.  usage: compute-sanitizer --tool T python
tools/sanitize_run.py"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import atfspec as A  # noqa: E402
from paper_conf_hpdc_raschg18_b200 import Space, _lib as L  # noqa: E402

SPECS = [A.c2_xgemm_direct(256), A.c3_xgemm("IS1"), A.c3_xgemm((20, 96, 8)), A.c5_chains(300, 4), A.c5_chains(4096, 2),
         A.saxpy(360)]
FLAGS = [0, L.ATF_FLAG_NO_SEG_BOUNDS, L.ATF_FLAG_NO_TAIL | L.ATF_FLAG_NO_JIT]

for spec in SPECS:
    for fl in FLAGS:
        with Space(spec, flags=fl) as sp:
            sp.generate()
            G = sp.num_groups()
            sizes = sp.group_sizes()
            n = 4096
            dig = torch.stack([torch.randint(0, max(1, z), (n,), device="cuda") for z in sizes])
            rows = sp.decode_digits(dig)
            back = sp.encode_digits(rows)
            assert torch.equal(back, dig), spec.name
            print(spec.name, fl, sp.size(), flush=True)
# int64-valued parameters (reading #22): generic kernels over int64 value tables, int64 decode
sys.path.insert(0, os.path.join(ROOT, "tests"))
from test_int64_values import mixed_groups64, wide64  # noqa: E402
for spec in (wide64(600, 120), mixed_groups64()):
    with Space(spec) as sp:
        sp.generate()
        sp.generate()
        S = sp.size()
        out = sp.decode(torch.arange(min(S, 8192), dtype=torch.int64, device="cuda"))
        assert out.dtype == torch.int64
        print(spec.name, S, flush=True)
torch.cuda.synchronize()
# balanced multi-GPU generation: two virtual ranks on their own streams, three generations
# (synchronous, log-sized, replay with device round flags)
from paper_conf_hpdc_raschg18_b200.shard import virtual_ranks  # noqa: E402
for spec in (A.c5_chains(4096, 4), A.c3_xgemm((20, 96, 8))):
    spaces = [Space(spec, flags=L.ATF_FLAG_NO_SEG_BOUNDS, stream=torch.cuda.Stream()) for _ in range(2)]
    for _ in range(3):
        virtual_ranks(spaces)
        print("dist", spec.name, [sp.group_sizes() for sp in spaces], flush=True)
    for sp in spaces:
        sp.close()
torch.cuda.synchronize()
print("sanitize run ok")
