"""CPU-side tests of the C ABI: the library loads and exports every symbol the headers
declare; the host planner (validation, static analysis, group partition, atom
compilation) behaves as documented.  No CUDA device is needed (no compute calls)."""
import os
import re
import subprocess

import pytest

import atfspec as A
from atfspec import Spec, X, C, P, interval, set_, divides
from oracle import run as orc

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def L():
    from paper_conf_hpdc_raschg18_b200 import _lib
    return _lib


def _declared(header):
    txt = open(os.path.join(ROOT, "include", header)).read()
    txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
    return set(re.findall(r"\b(atf_\w+)\s*\(", txt)) - {"atf_alloc_fn", "atf_free_fn"}


def test_library_exports_every_declared_symbol(L):
    declared = _declared("atfgen.h") | _declared("atfgen_test.h")
    assert declared, "no declarations parsed"
    out = subprocess.run(["nm", "-D", "--defined-only", L.LIB_PATH], capture_output=True, text=True).stdout
    exported = set(re.findall(r" T (atf_\w+)", out))
    assert declared <= exported, declared - exported
    assert declared <= set(L.EXPORTED) | {"atf_test_exclusive_scan_u32"}
    for name in declared:
        assert hasattr(L, name)


def test_library_is_sm100a(L):
    out = subprocess.run(["cuobjdump", "--list-elf", L.LIB_PATH], capture_output=True, text=True).stdout
    assert "sm_100a" in out


def _space(spec, **kw):
    from paper_conf_hpdc_raschg18_b200 import Space
    return Space(spec, torch_alloc=False, **kw)


@pytest.mark.parametrize("mk", [A.fig1, A.c1_toy, lambda: A.c2_xgemm_direct(64), lambda: A.c3_xgemm("IS3"),
                                lambda: A.c5_chains(32, 4)] + [lambda s=s: A.random_spec(s) for s in range(25)])
def test_group_partition_matches_oracle(oracle_bin, mk):
    spec = mk()
    sp = _space(spec)
    sp.plan()
    try:
        ref = orc.info(spec)
    except ValueError:
        return
    assert sp.groups() == [g["members"] for g in ref["groups"]]


def test_named_partitions():
    # SURVEY.md §8(a) A2
    for spec, want in [(A.fig1(), [[0, 1], [2, 3]]), (A.c2_xgemm_direct(256), [list(range(8)), [8], [9]]),
                       (A.c3_xgemm("IS2"), [list(range(10)), [10], [11], [12], [13]]),
                       (A.c5_chains(), [list(range(8)), list(range(8, 16)), list(range(16, 24))])]:
        sp = _space(spec)
        sp.plan()
        assert sp.groups() == want


def test_atoms_for_the_hot_levels():
    """The C3 NDIMB level (the dominant one) compiles to the divisibility
    atom x|NWG and the computed-divisor atom KWG mod (MDIMC*NDIMC/x) == 0, both 16-bit."""
    sp = _space(A.c3_xgemm("IS2"))
    sp.plan()
    lv = sp.plan_json()["groups"][0]["levels"]
    kinds = [[t["kind"] for t in l["terms"]] for l in lv]
    assert kinds[6] == [2, 5] and all(t["variant"] == 0 for t in lv[6]["terms"])
    assert lv[6]["terms"][1]["qtable"] == 0  # quotient divisibility divides inline
    assert kinds[8] == [4, 4] and kinds[9] == [4, 4]
    assert lv[6]["cost"] == 9.0 and lv[9]["cost"] == 5.0
    sp = _space(A.c5_chains())
    sp.plan()
    pj = sp.plan_json()
    assert all(l["terms"][0]["kind"] == (2 if g != 1 else 3) for g in range(3)
               for l in pj["groups"][g]["levels"][1:])
    assert [g["words"] for g in pj["groups"]] == [4, 4, 4]


def test_generic_only_flag_compiles_generic_terms(L):
    sp = _space(A.c3_xgemm("IS2"), flags=L.ATF_FLAG_GENERIC_ONLY)
    sp.plan()
    lv = sp.plan_json()["groups"][0]["levels"]
    assert all(t["kind"] == 6 for l in lv for t in l["terms"])


def test_record_packing_two_words():
    sp = _space(A.c3_xgemm("IS2"))
    sp.plan()
    g0 = sp.plan_json()["groups"][0]
    assert g0["words"] == 2        # 59 bits packed first-fit-decreasing into two words
    used = {}
    for l in g0["levels"]:
        used.setdefault(l["word"], []).append((l["shift"], l["bits"]))
    for w, fields in used.items():
        fields.sort()
        for (s0, b0), (s1, _) in zip(fields, fields[1:]):
            assert s0 + b0 <= s1
        assert fields[-1][0] + fields[-1][1] <= 32


def _err(fn):
    from paper_conf_hpdc_raschg18_b200 import AtfError
    with pytest.raises(AtfError) as e:
        fn()
    return e.value.status


def test_validation_errors():
    from paper_conf_hpdc_raschg18_b200 import Space
    sp = Space(None, torch_alloc=False)
    a = sp.add_param("a", interval(1, 8))
    b = sp.add_param("b", interval(1, 8))
    assert _err(lambda: sp.add_param("a", interval(1, 2))) == -9                    # duplicate name
    assert _err(lambda: sp.add_param("s", set_(1, 2, 2))) == -9                      # duplicate set value
    assert _err(lambda: sp.add_param("t", {"kind": "interval", "begin": 1, "end": 4, "step": 0})) == -1
    assert _err(lambda: sp.add_param("u", {"kind": "pow2", "begin": 0, "end": 63, "step": 1})) == -1  # 2^63 > int64
    assert _err(lambda: sp.add_constraint(a, P(1).code + [1, 17])) == -6           # forward reference
    assert _err(lambda: sp.add_constraint(b, [1, 17])) == -5                         # stack underflow
    assert _err(lambda: sp.add_constraint(b, [1, 1])) == -5                          # two results
    assert _err(lambda: sp.add_constraint(b, [99])) == -5                            # bad opcode
    assert _err(lambda: sp.add_constraint(b, [1] * 17 + [4] * 16)) == -5           # depth > 16
    sp.add_constraint(b, divides(P(a)).code)
    assert _err(lambda: sp.size()) == -4                                             # state
    sp.plan()
    assert _err(lambda: sp.add_param("c", interval(1, 2))) == -4
    assert sp.groups() == [[0, 1]]


def test_static_overflow_rejected():
    s = Spec("ovf")
    s.add("x", interval(1, 4), (C(2 ** 62) * X) > 0)
    sp = _space(s)
    assert _err(sp.plan) == -7
    s = Spec("ok")
    s.add("x", interval(1, 4), (C(2 ** 60) * X) > 0)
    _space(s).plan()


def test_magic_formulas_exhaustive(tmp_path):
    """The kernel's divisibility / quotient magics (Lemire, Kaser & Kurz 2019) restated in C and
    checked exhaustively over all 16-bit pairs and on random 32-bit pairs against % and /.
    Includes the wide kernel's hot filter: for 16-bit n and d, (n * ceil(2^32/d) mod 2^32) <
    2^16 iff d | n, which lets the hot loop take a min over candidates against one bound."""
    src = tmp_path / "magic.c"
    src.write_text(r'''
#include <stdint.h>
#include <stdio.h>
int main(void) {
  unsigned long long bad = 0;
  for (uint32_t d = 1; d < 65536; d++) {
    uint32_t m = 0xffffffffu / d + 1u;            /* ceil(2^32/d) mod 2^32 */
    for (uint32_t n = 0; n < 65536; n++) {
      int div = (uint32_t)(n * m) <= m - 1u;       /* V16 divisibility test */
      int hot = (uint32_t)(n * m) < 65536u;         /* wide kernel's HOT_DIVX filter: uniform bound */
      uint32_t q = d == 1 ? n : (uint32_t)(((uint64_t)n * m) >> 32);  /* V16 quotient */
      bad += (div != (n % d == 0)) + (hot != (n % d == 0)) + (q != n / d);
    }
  }
  uint64_t s = 88172645463325252ull;
  for (int i = 0; i < 20000000; i++) {
    s ^= s << 13; s ^= s >> 7; s ^= s << 17;
    uint32_t n = (uint32_t)s, d = (uint32_t)(s >> 32) >> (s & 31);
    if (!d) d = 1;
    uint64_t m = ~0ull / d + 1ull;                 /* ceil(2^64/d) mod 2^64 */
    int div = (uint64_t)n * m <= m - 1ull;         /* V32 divisibility test */
    uint64_t q = d == 1 ? n : (uint64_t)(((unsigned __int128)m * n) >> 64);  /* V32 quotient */
    bad += (div != (n % d == 0)) + (q != n / d);
  }
  printf("%llu\n", bad);
  return 0;
}
''')
    exe = tmp_path / "magic"
    subprocess.check_call(["gcc", "-O2", "-o", str(exe), str(src)])
    assert subprocess.check_output([str(exe)], timeout=300).strip() == b"0"


def test_generator_range_abi_validation(L):
    """The library materialises generator ranges on the host (no GPU needed): duplicates,
    zero divisors, PARAM references and non-int32 values are rejected."""
    import ctypes as C
    from paper_conf_hpdc_raschg18_b200 import _lib as LL

    def add(expr_code, b, e, step=1):
        sp = C.c_void_p()
        LL.check(LL.atf_space_create(None, C.byref(sp)))
        try:
            code = (C.c_int32 * len(expr_code))(*expr_code)
            r = LL.atf_range(LL.ATF_RANGE_GEN, b, e, step, C.cast(code, C.POINTER(C.c_int32)), len(expr_code))
            pid = C.c_int32()
            return LL.atf_space_add_param(sp, b"p", C.byref(r), C.byref(pid))
        finally:
            LL.atf_space_destroy(sp)
    assert add(A.gen(1, 10, A.X * A.X)["code"], 1, 10) == 0
    assert add(A.gen(-2, 2, A.X * A.X)["code"], -2, 2) == -9           # duplicate
    assert add(A.gen(0, 3, A.C(12) // A.X)["code"], 0, 3) == -5         # 12 / 0: poison
    assert add([2, 0], 0, 3) == -5                                       # PARAM 0
    assert add(A.gen(0, 3, A.X * A.C(1 << 40))["code"], 0, 3) == 0      # int64 values (reading #22)
    assert add(A.gen(0, 3, A.X * A.C(1 << 62))["code"], 0, 3) == -7     # > int64: overflow


def test_jit_level_sources_compile_for_sm100a(L, tmp_path):
    """Narrow fast levels are specialised at run time (jit.cpp, NVRTC on the GPU box); here the
    generated sources of every C1-C3 narrow level (+ fuzz specs) compile with nvcc for sm_100a."""
    import ctypes as C
    from paper_conf_hpdc_raschg18_b200 import _lib as LL
    specs = [A.c1_toy(), A.c2_xgemm_direct(256), A.c3_xgemm("IS2"), A.c3_xgemm("IS4"), A.saxpy(360)]
    specs += [A.random_spec(s) for s in range(0, 40, 3)]
    srcs, tails = [], []
    for spec in specs:
        sp = C.c_void_p()
        LL.check(LL.atf_space_create(None, C.byref(sp)))
        try:
            keep = []
            for p in spec.params:
                from paper_conf_hpdc_raschg18_b200.space import _range_struct
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
                    srcs.append(buf.value.decode())
                    tails.append((spec.name, g, k0.value))
                nl = C.c_int32()
                LL.check(LL.atf_space_num_levels(sp, g, C.byref(nl)), sp)
                for k in range(nl.value):
                    n = C.c_size_t()
                    LL.check(LL.atf_test_jit_source(sp, g, k, None, 0, C.byref(n)), sp)
                    if n.value:
                        buf = C.create_string_buffer(n.value + 1)
                        LL.check(LL.atf_test_jit_source(sp, g, k, buf, n.value + 1, None), sp)
                        srcs.append(buf.value.decode())
        finally:
            LL.atf_space_destroy(sp)
    assert len(srcs) >= 6
    # fused narrow tails: C2's VWMD/VWND, C3-IS2's KWI/VWM/VWN, C3-IS4's KWI (r = 64: u64 masks,
    # NVRTC tail only) / VWM / VWN
    assert ("C2_xgemm_direct_256", 0, 6) in tails and ("C3_xgemm_IS2", 0, 7) in tails
    assert ("C3_xgemm_IS4", 0, 7) in tails
    assert any("u64 tmask0" in x for x in srcs)
    # mid-width levels (C2's WGD..KWID, C3's NWG / NDIMC / NDIMB, r = 256..576): exact-mask kernels
    assert sum("atf_wide_jit" in x for x in srcs) >= 8
    # one translation unit per source (kernel names collide), compiled in parallel
    procs = []
    for i, src in enumerate(srcs):
        f = tmp_path / f"lvl{i}.cu"
        f.write_text(src)
        procs.append(subprocess.Popen(["/usr/local/cuda/bin/nvcc", "-gencode", "arch=compute_100a,code=sm_100a",
                                       "-std=c++17", "-c", str(f), "-o", str(tmp_path / f"lvl{i}.o")],
                                      stdout=subprocess.PIPE, stderr=subprocess.STDOUT, text=True))
        if len(procs) >= 8:
            for p in procs:
                out, _ = p.communicate()
                assert p.returncode == 0, out
            procs = []
    for p in procs:
        out, _ = p.communicate()
        assert p.returncode == 0, out


def test_new_entry_points_validate_without_a_gpu(L):
    """encode / neighbours before generate -> ATF_ERR_STATE; the full-product filter of a
    product >= 2^64 -> ATF_ERR_OVERFLOW; bad arguments -> ATF_ERR_INVALID_ARG (no CUDA work)."""
    import ctypes as C
    from paper_conf_hpdc_raschg18_b200 import _lib as LL
    from paper_conf_hpdc_raschg18_b200.space import _range_struct
    sp = C.c_void_p()
    LL.check(LL.atf_space_create(None, C.byref(sp)))
    try:
        keep = []
        for i in range(5):  # 5 parameters of 2^14 values: product 2^70
            rs, k = _range_struct(A.interval(1, 1 << 14))
            keep.append(k)
            pid = C.c_int32()
            LL.check(LL.atf_space_add_param(sp, f"p{i}".encode(), C.byref(rs), C.byref(pid)), sp)
        dummy = C.c_void_p(16)
        assert LL.atf_space_encode_digits(sp, dummy, 4, 4, dummy, None) == -4      # STATE
        assert LL.atf_space_encode_indices(sp, dummy, 4, 4, dummy, dummy, None) == -4
        assert LL.atf_space_neighbors(sp, dummy, 4, 4, 1, 8, dummy, 4, dummy, None) == -4
        assert LL.atf_space_encode_digits(sp, None, 4, 4, dummy, None) == -1       # INVALID_ARG
        assert LL.atf_space_neighbors(sp, dummy, 2, 4, 1, 8, dummy, 4, dummy, None) == -1  # ld < n
        cnt, tot = C.c_uint64(), C.c_uint64()
        assert LL.atf_space_filter_product(sp, C.byref(cnt), C.byref(tot)) == -7  # OVERFLOW
    finally:
        LL.atf_space_destroy(sp)


def test_float_parameters_are_monotone_positions():
    """NEXT-3 floats by position (atfspec.floats / float_interval): positions 0..n-1 in the listed
    order; for an interval, position order = value order, so X <= float_code(v) selects the
    values <= v; the oracle enumerates the positions like any SET."""
    from oracle import run as orc
    r = A.float_interval(0.1, 1.0, 0.1)
    assert len(r["values"]) == 10 and r["values"] == list(range(10))
    vals = r["names"]
    assert all(a < b for a, b in zip(vals, vals[1:]))
    s = A.Spec("f")
    s.add("t", r, A.X <= A.float_code(r, vals[4]))
    d, rows = orc.o1(s)
    assert [vals[int(x)] for x in rows[:, 0]] == [v for v in vals if v <= vals[4]]
    with pytest.raises(ValueError):
        A.floats(0.5, 0.5)
