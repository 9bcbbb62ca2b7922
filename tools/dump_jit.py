"""Write the NVRTC sources the planner generates for a spec (fused tails and narrow/wide levels)
to a directory, for reading ncu source-page line numbers:  python tools/dump_jit.py C3-IS2 outdir"""
import ctypes as C
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import atfspec as A  # noqa: E402
from paper_conf_hpdc_raschg18_b200 import _lib as LL  # noqa: E402
from paper_conf_hpdc_raschg18_b200.space import _range_struct  # noqa: E402

NAMED = {"C1": A.c1_toy, "C2": lambda: A.c2_xgemm_direct(256), "C3-IS1": lambda: A.c3_xgemm("IS1"),
         "C3-IS2": lambda: A.c3_xgemm("IS2"), "C3-IS3": lambda: A.c3_xgemm("IS3"), "C3-IS4": lambda: A.c3_xgemm("IS4"),
         "C5": lambda: A.c5_chains(4096, 8)}
spec = NAMED[sys.argv[1]]()
out = sys.argv[2]
os.makedirs(out, exist_ok=True)
sp = C.c_void_p()
LL.check(LL.atf_space_create(None, C.byref(sp)))
keep = []
for p in spec.params:
    rs, k = _range_struct(p.range)
    keep.append(k)
    pid = C.c_int32()
    LL.check(LL.atf_space_add_param(sp, p.name.encode(), C.byref(rs), C.byref(pid)), sp)
    for code in p.constraints:
        arr = (C.c_int32 * len(code))(*code)
        LL.check(LL.atf_space_add_constraint(sp, pid.value, arr, len(code)), sp)
LL.check(LL.atf_space_plan(sp), sp)
G = C.c_int32()
LL.check(LL.atf_space_num_groups(sp, C.byref(G)), sp)
for g in range(G.value):
    n, k0 = C.c_size_t(), C.c_int32()
    LL.check(LL.atf_test_tail_source(sp, g, None, 0, C.byref(n), C.byref(k0)), sp)
    if n.value:
        buf = C.create_string_buffer(n.value + 1)
        LL.check(LL.atf_test_tail_source(sp, g, buf, n.value + 1, None, None), sp)
        open(f"{out}/g{g}_tail_k{k0.value}.cu", "w").write(buf.value.decode())
    nl = C.c_int32()
    LL.check(LL.atf_space_num_levels(sp, g, C.byref(nl)), sp)
    for k in range(nl.value):
        n = C.c_size_t()
        LL.check(LL.atf_test_jit_source(sp, g, k, None, 0, C.byref(n)), sp)
        if n.value:
            buf = C.create_string_buffer(n.value + 1)
            LL.check(LL.atf_test_jit_source(sp, g, k, buf, n.value + 1, None), sp)
            open(f"{out}/g{g}_l{k}.cu", "w").write(buf.value.decode())
LL.atf_space_destroy(sp)
print("\n".join(sorted(os.listdir(out))))
