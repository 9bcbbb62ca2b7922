"""int64-valued parameter ranges ("a range of values of an
arbitrary fundamental type T (e.g., bool, integer, or float)"; reading #22).

CPU part: pins of the oracle on spaces whose values do not fit int32 — closed forms
(multiplicative divisor sums, counts of multiples in an interval) and brute force written out in
Python on tiny inputs (never the oracle against itself).  GPU part (`-m gpu`): the library's
generation and its int64 decoders against the oracle, element by element.
"""
import itertools

import numpy as np
import pytest

import atfspec as A
from atfspec import C, P, Spec, X, divides, interval, pow2, set_
from oracle import run as orc

# ---------------------------------------------------------------- specs
N64 = 2 ** 35 * 3 ** 2 * 5          # 1,546,188,226,560 > 2^31
B64 = 2 ** 33 + 7                    # interval start above 2^32
EDGE = [2 ** 31 - 1, 2 ** 31, 2 ** 32, -(2 ** 31) - 1, 5, -(2 ** 40), 2 ** 40 + 3]


def divisors_by_exponents():
    """Divisors of N64 = 2^35 3^2 5 from its exponents (ascending)."""
    return sorted(2 ** a * 3 ** b * 5 ** c for a in range(36) for b in range(3) for c in range(2))


def saxpy64():
    """P:41/P:49/P:59 saxpy constraints at N = N64: WPT | N, LS | N / WPT, over the divisors."""
    d = divisors_by_exponents()
    s = Spec("saxpy64")
    s.add("WPT", set_(*d), divides(N64))
    s.add("LS", set_(*d), divides(C(N64) // P(0)))
    return s


def pow2_pairs(k=40):
    s = Spec("pow2pairs")
    s.add("a", pow2(0, k), divides(2 ** k))
    s.add("b", pow2(0, k), divides(C(2 ** k) // P(0)))
    return s


def interval_multiples(b0=B64, n=1000, m=64):
    s = Spec("ivmul64")
    s.add("x", interval(b0, b0 + n - 1))
    s.add("y", interval(1, m), divides(P(0)))
    return s


def edge_order():
    s = Spec("edge64")
    s.add("x", set_(*EDGE))
    s.add("y", set_(*EDGE), X > P(0))
    s.add("z", set_(*EDGE), X.eq(P(1)) | (X < P(0)))
    return s


def products64():
    vals = [2 ** 20, 2 ** 21, 3 * 2 ** 20, 2 ** 30 + 1, 7]
    s = Spec("prod64")
    s.add("x", set_(*vals))
    s.add("y", set_(*vals), (P(0) * X) <= 2 ** 41)
    s.add("w", interval(1, 12), divides(P(1)) | divides(P(0)))
    return s, vals


def mixed_groups64():
    """Two groups: an int64 chain and an int32 pair (mixed widths in one space)."""
    s = Spec("mixed64")
    s.add("t", set_(2 ** 36, 2 ** 34 * 3, 10 ** 11, 7))
    s.add("u", interval(1, 40), divides(P(0)))
    s.add("v", pow2(30, 36), divides(P(0)) | (X > P(1)))
    s.add("p", interval(1, 12))
    s.add("q", interval(1, 12), divides(P(3)))
    return s


def fuzz64(seed):
    """Seeded random int64 specs: 3-4 parameters, small sets mixing int32 and int64 values,
    divisibility / order / equality constraints on earlier parameters (no products of two
    int64 values, which the static overflow analysis would reject)."""
    rng = np.random.default_rng(seed)
    s = Spec(f"fuzz64_{seed}")
    n = int(rng.integers(3, 5))
    for p in range(n):
        r = int(rng.integers(2, 9))
        pool = set()
        while len(pool) < r:
            kind = int(rng.integers(0, 4))
            if kind == 0:
                v = int(rng.integers(-20, 21))
            elif kind == 1:
                v = int(rng.integers(1, 1 << 12)) << int(rng.integers(20, 40))
            elif kind == 2:
                v = -int(rng.integers(1, 1 << 20)) << int(rng.integers(12, 30))
            else:
                v = int(rng.choice([2 ** 31 - 1, 2 ** 31, -(2 ** 31), 2 ** 32, 2 ** 32 + 1, 6 * 2 ** 33]))
            pool.add(v)
        vals = list(pool)
        rng.shuffle(vals)
        cons = None
        if p > 0:
            j = int(rng.integers(0, p))
            c = int(rng.integers(0, 5))
            if c == 0:
                cons = divides(P(j))
            elif c == 1:
                cons = A.is_multiple_of(P(j))
            elif c == 2:
                cons = X < P(j)
            elif c == 3:
                cons = X.ne(P(j)) & (X > -(2 ** 35))
            else:
                cons = divides(P(j)) | (X >= P(j))
        s.add(f"p{p}", set_(*vals), *( [cons] if cons is not None else []))
    return s


def _values(spec):
    """Materialised ranges of the specs above (sets / intervals / pow2 only), in range order."""
    out = []
    for prm in spec.params:
        r = prm.range
        if r["kind"] == "set":
            out.append(list(r["values"]))
        elif r["kind"] == "interval":
            out.append(list(range(r["begin"], r["end"] + 1, r["step"])))
        elif r["kind"] == "pow2":
            out.append([2 ** i for i in range(r["begin"], r["end"] + 1, r["step"])])
        else:
            raise ValueError(r["kind"])
    return out


# ---------------------------------------------------------------- oracle pins (CPU)
def test_width_flag(oracle_bin):
    assert orc.width(saxpy64()) and orc.width(pow2_pairs()) and orc.width(edge_order())
    assert not orc.width(A.saxpy(64)) and not orc.width(A.c1_toy())
    assert not orc.width(pow2_pairs(30))   # 2^30 still fits int32


def test_saxpy64_multiplicative_closed_form(oracle_bin):
    """S = sum_{d|N} tau(d) = prod_p (a_p+1)(a_p+2)/2 for N = 2^35 3^2 5: 666 * 6 * 3 = 11,988;
    f_1 = tau(N) = 36 * 3 * 2 = 216 (P:41, P:49, P:59 at a size beyond int32)."""
    d = orc.info(saxpy64())
    assert int(d["S"]) == 666 * 6 * 3 == 11988
    assert [lv["f"] for lv in d["groups"][0]["levels"]] == [216, 11988]
    assert d["overflow"] is False


def test_pow2_pairs_closed_form_and_rows(oracle_bin):
    """a, b in {2^0..2^40}, a | 2^40, b | 2^40 / a: pairs (2^i, 2^j) with i + j <= 40 ->
    41 * 42 / 2 = 861 rows, in range-position order (reading #4); the rows are the exact
    int64 values (a truncating writer would print 0 for 2^32)."""
    spec = pow2_pairs()
    d = orc.info(spec)
    assert int(d["S"]) == 41 * 42 // 2
    want = np.array([(2 ** i, 2 ** j) for i in range(41) for j in range(41) if i + j <= 40], dtype=np.int64)
    rows = orc.leaves(spec, 0, 2)
    assert rows.dtype == np.int64 and np.array_equal(rows, want)
    _, o1rows = orc.o1(spec)
    assert np.array_equal(o1rows, want)


@pytest.mark.parametrize("b0", [B64, -(2 ** 35) - 3, 2 ** 62 - 500])
def test_interval_multiples_count(oracle_bin, b0):
    """x in [b0, b0+999] (int64 interval, reading #1), y in [1,64], y | x:
    count = sum_y floor((b0+999)/y) - floor((b0-1)/y) (multiples of y in the interval)."""
    d = orc.info(interval_multiples(b0))
    want = sum((b0 + 999) // y - (b0 - 1) // y for y in range(1, 65))
    assert int(d["S"]) == want
    assert [lv["f"] for lv in d["groups"][0]["levels"]] == [1000, want]


def test_edge_values_brute_force(oracle_bin):
    """Order and equality across the int32 boundary, brute force in Python: (x, y, z) with
    y > x and (z == y or z < x)."""
    spec = edge_order()
    vals = EDGE
    want = [(x, y, z) for x in vals for y in vals if y > x for z in vals if z == y or z < x]
    _, rows = orc.o1(spec)
    assert rows.dtype == np.int64
    assert [tuple(r) for r in rows.tolist()] == want


def test_products_brute_force(oracle_bin):
    """x * y <= 2^41 with int64 products; w | y or w | x (brute force in Python)."""
    spec, vals = products64()
    want = [(x, y, w) for x in vals for y in vals if x * y <= 2 ** 41
            for w in range(1, 13) if y % w == 0 or x % w == 0]
    _, rows = orc.o1(spec)
    assert [tuple(r) for r in rows.tolist()] == want
    assert int(orc.info(spec)["S"]) == len(want)


def test_mixed_groups_brute_force(oracle_bin):
    spec = mixed_groups64()
    d = orc.info(spec)
    assert [g["members"] for g in d["groups"]] == [[0, 1, 2], [3, 4]]
    tv = [2 ** 36, 2 ** 34 * 3, 10 ** 11, 7]
    g0 = [(t, u, v) for t in tv for u in range(1, 41) if t % u == 0
          for v in [2 ** k for k in range(30, 37)] if t % v == 0 or v > u]
    g1 = [(p, q) for p in range(1, 13) for q in range(1, 13) if p % q == 0]
    assert [g["size"] for g in d["groups"]] == [len(g0), len(g1)]
    assert [tuple(r) for r in orc.leaves(spec, 0, 3).tolist()] == g0
    # decode: group 0 most significant (reading #11), every index
    S = len(g0) * len(g1)
    _, soa = orc.decode(spec, np.arange(S, dtype=np.uint64))
    assert soa.dtype == np.int64
    want = np.array([g0[i // len(g1)] + g1[i % len(g1)] for i in range(S)], dtype=np.int64).T
    assert np.array_equal(soa, want)


@pytest.mark.parametrize("seed", range(12))
def test_fuzz64_o1_equals_o2_and_python(oracle_bin, seed):
    """Random int64 specs: O1 (full product) == O2 (pruned) == a Python brute force restating the
    opcode semantics (reading #6/#7) on the materialised ranges."""
    spec = fuzz64(seed)
    vals = _values(spec)
    d = orc.info(spec, hash=True)
    _, rows = orc.o1(spec)
    assert int(d["S"]) == rows.shape[0]
    # Python brute force over the product (declaration order), each constraint restated
    def ok(prm, x, row):
        for code in prm.constraints:
            if not _py_eval(code, x, row):
                return False
        return True
    want = []
    for tup in itertools.product(*vals):
        if all(ok(spec.params[p], tup[p], tup) for p in range(len(vals))):
            want.append(tup)
    # canonical order: group-major range positions (groups = connected components)
    pos = [{v: i for i, v in enumerate(vs)} for vs in vals]
    members = [g["members"] for g in d["groups"]]
    want.sort(key=lambda t: [pos[q][t[q]] for g in members for q in g])
    assert [tuple(r) for r in rows.tolist()] == want
    for g, mem in enumerate(members):
        leaves = orc.leaves(spec, g, len(mem))
        assert orc.rowhash_rows(leaves, w64=orc.width(spec)) == int(d["groups"][g]["hash"])


def _py_eval(code, x, row):
    """SURVEY.md §8(b) postfix semantics, restated in Python (exact integers, C truncation,
    zero divisor = poison -> reject)."""
    st = []
    i = 0
    while i < len(code):
        op = code[i]
        if op == 1:
            st.append(x); i += 1; continue
        if op == 2:
            st.append(row[code[i + 1]]); i += 2; continue
        if op == 3:
            lo, hi = code[i + 1] & 0xFFFFFFFF, code[i + 2] & 0xFFFFFFFF
            v = (hi << 32) | lo
            st.append(v - (1 << 64) if v >= 1 << 63 else v); i += 3; continue
        if op == 21:
            st[-1] = int(st[-1] == 0); i += 1; continue
        b = st.pop(); a = st.pop()
        def tdiv(p, q):
            r = abs(p) // abs(q)
            return r if (p >= 0) == (q >= 0) else -r
        if (op == 17 and a == 0) or (op in (7, 8, 18) and b == 0):
            return False   # zero divisor: poison rejects the candidate (reading #7)
        r = {4: lambda: a + b, 5: lambda: a - b, 6: lambda: a * b,
             7: lambda: tdiv(a, b), 8: lambda: a - tdiv(a, b) * b,
             9: lambda: min(a, b), 10: lambda: max(a, b),
             11: lambda: int(a == b), 12: lambda: int(a != b), 13: lambda: int(a < b),
             14: lambda: int(a <= b), 15: lambda: int(a > b), 16: lambda: int(a >= b),
             17: lambda: int(b % a == 0), 18: lambda: int(a % b == 0),
             19: lambda: int(a != 0 and b != 0), 20: lambda: int(a != 0 or b != 0)}[op]()
        st.append(r)
        i += 1
    return len(st) == 1 and st[0] != 0


def test_check_int64_rows(oracle_bin):
    """check on int64 rows: every O1 row valid; a row whose int64 value is replaced by
    its int32 truncation (2^36 -> 0, 2^34*3 -> 0) is outside the range and invalid."""
    spec = mixed_groups64()
    _, rows = orc.o1(spec)
    assert orc.check(spec, rows)["valid"] == rows.shape[0]
    bad = rows[:50].copy()
    bad[:, 0] = bad[:, 0].astype(np.int32).astype(np.int64)
    assert orc.check(spec, bad)["valid"] == int(np.sum(rows[:50, 0] == 7))


def test_overflow_int64_values(oracle_bin):
    """Exact int64 arithmetic (reading #9): 2^62 * x overflows for x = 2^62."""
    s = Spec("ovf64"); s.add("x", set_(2 ** 62, 3), (X * X) > 0)
    assert orc.info(s)["overflow"] is True


# ---------------------------------------------------------------- library host side (CPU)
def _lib_space(spec, **kw):
    from paper_conf_hpdc_raschg18_b200 import Space
    return Space(spec, torch_alloc=False, **kw)


def _status(fn):
    from paper_conf_hpdc_raschg18_b200 import AtfError
    with pytest.raises(AtfError) as e:
        fn()
    return e.value.status


def test_library_value_bits_and_generic_levels():
    """An int64 parameter's own level is compiled to generic (interpreted, int64) terms; the
    int32 group of the same space keeps its divisibility atoms (plan_json kinds: 2 = x | n,
    6 = generic)."""
    assert _lib_space(A.c1_toy()).value_bits() == 32
    sp = _lib_space(mixed_groups64())
    assert sp.value_bits() == 64
    sp.plan()
    pj = sp.plan_json()
    g0, g1 = pj["groups"]
    assert all(t["kind"] == 6 for t in g0["levels"][0]["terms"] + g0["levels"][2]["terms"])
    assert [t["kind"] for t in g1["levels"][1]["terms"]] == [2]
    assert _lib_space(pow2_pairs(30)).value_bits() == 32


def test_library_int64_range_validation():
    from paper_conf_hpdc_raschg18_b200 import Space
    sp = Space(None, torch_alloc=False)
    sp.add_param("a", pow2(0, 62))
    assert _status(lambda: sp.add_param("b", pow2(0, 63))) == -1                 # 2^63 outside int64
    assert _status(lambda: sp.add_param("c", set_(2 ** 40, 5, 2 ** 40))) == -9   # duplicate (reading #5)
    sp.add_param("d", interval(2 ** 62, 2 ** 62 + 10))
    sp.add_param("e", A.gen(0, 3, X * (2 ** 40)))
    sp.add_param("f", set_(-(2 ** 63), 2 ** 63 - 1))
    assert sp.value_bits() == 64
    s = Spec("ovf64"); s.add("x", set_(2 ** 62, 3), (X * X) > 0)
    assert _status(_lib_space(s).plan) == -7   # static analysis: int64 overflow (reading #9)


def test_library_int32_entry_points_refuse_int64_spaces():
    sp = _lib_space(mixed_groups64())
    assert _status(sp.filter_product) == -10


# ---------------------------------------------------------------- GPU parity (-m gpu)
def wide64(n_x=5000, n_y=300):
    """An int64 level with r > 64 over a frontier of several warp tiles with a ragged tail
    (the warp-tile kernel's dense path), and an int32 level reading an int64 ancestor
    (64-bit atoms, generic kernels): y_j = j * 2^33 (j = 1..n_y), y / 2^33 a multiple of x;
    z | y / 2^33 with z in 1..96."""
    s = Spec(f"wide64_{n_x}x{n_y}")
    s.add("x", interval(1, n_x))
    s.add("y", set_(*[j * 2 ** 33 for j in range(1, n_y + 1)]), A.is_multiple_of(P(0) * 2 ** 33))
    s.add("z", interval(1, 96), divides(P(1) // 2 ** 33))
    return s


GPU_SPECS = {
    "saxpy64": saxpy64, "pow2pairs": pow2_pairs, "ivmul64": interval_multiples,
    "ivmul64neg": lambda: interval_multiples(-(2 ** 35) - 3), "ivmul64top": lambda: interval_multiples(2 ** 62 - 500),
    "edge64": edge_order, "prod64": lambda: products64()[0], "mixed64": mixed_groups64, "wide64": wide64,
}


@pytest.fixture(scope="module")
def GSpace():
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_hpdc_raschg18_b200 import Space as S
    return S


def _gpu_check(Space, spec, flags=0, regenerate=False):
    import torch
    ref = orc.info(spec, threads=8)
    with Space(spec, flags=flags) as sp:
        sp.generate()
        if regenerate:          # replay, then the CUDA graph capture and its launch
            for _ in range(3):
                sp.generate()
        assert sp.value_bits() == (64 if orc.width(spec) else 32)
        assert sp.groups() == [g["members"] for g in ref["groups"]]
        assert sp.size() == int(ref["S"])
        for g, grp in enumerate(ref["groups"]):
            assert sp.level_sizes(g) == [lv["f"] for lv in grp["levels"]], (spec.name, g)
        S = sp.size()
        if S == 0:
            return
        idx = torch.arange(S, dtype=torch.int64, device="cuda")
        got = sp.decode(idx, out=torch.empty((len(spec.params), S), dtype=torch.int64, device="cuda"))
        _, want = orc.decode(spec, np.arange(S, dtype=np.uint64))
        assert np.array_equal(got.cpu().numpy(), want), spec.name
        # decode_range (u128 path) over a window and decode_digits of group 0's leaves
        n = min(S, 4096)
        first = S - n
        assert np.array_equal(sp.decode_range(first, n).cpu().numpy(), want[:, first:])
        G = sp.num_groups()
        sz0 = sp.group_sizes()[0]
        dig = torch.zeros((G, sz0), dtype=torch.int64, device="cuda")
        dig[0] = torch.arange(sz0, dtype=torch.int64, device="cuda")
        lv = sp.decode_digits(dig)[ref["groups"][0]["members"]].T.cpu().numpy()
        assert np.array_equal(lv, orc.leaves(spec, 0, len(ref["groups"][0]["members"])))


@pytest.mark.gpu
@pytest.mark.parametrize("name", sorted(GPU_SPECS))
def test_gpu_int64_named(GSpace, name):
    _gpu_check(GSpace, GPU_SPECS[name]())


@pytest.mark.gpu
@pytest.mark.parametrize("seed", range(12))
def test_gpu_int64_fuzz(GSpace, seed):
    spec = fuzz64(seed)
    if not orc.width(spec):
        pytest.skip("draw without int64 values")
    _gpu_check(GSpace, spec)


@pytest.mark.gpu
@pytest.mark.parametrize("variant", ["legacy_wide", "no_replay_regen", "regen", "no_seg_bounds"])
def test_gpu_int64_flags(GSpace, variant):
    from paper_conf_hpdc_raschg18_b200 import _lib as L
    flags = {"legacy_wide": L.ATF_FLAG_LEGACY_WIDE, "no_replay_regen": L.ATF_FLAG_NO_REPLAY,
             "regen": 0, "no_seg_bounds": L.ATF_FLAG_NO_SEG_BOUNDS}[variant]
    for spec in (wide64(), mixed_groups64()):
        _gpu_check(GSpace, spec, flags=flags, regenerate=variant.endswith("regen"))


@pytest.mark.gpu
def test_gpu_int64_errors(GSpace):
    """The int32 decoders and encode refuse an int64 space (ATF_ERR_OVERFLOW / ATF_ERR_LIMIT);
    out-of-range indices give INT64_MIN rows and ATF_ERR_INDEX; the int64 decoders sign-extend
    an int32 space's values."""
    import torch
    from paper_conf_hpdc_raschg18_b200 import AtfError
    from paper_conf_hpdc_raschg18_b200 import _lib as L
    spec = mixed_groups64()
    with GSpace(spec) as sp:
        sp.generate()
        S = sp.size()
        idx = torch.tensor([0, S, S - 1], dtype=torch.int64, device="cuda")
        with pytest.raises(AtfError) as e:
            sp.decode(idx, out=torch.empty((5, 3), dtype=torch.int32, device="cuda"))
        assert e.value.status == -7
        out = torch.empty((5, 3), dtype=torch.int64, device="cuda")
        with pytest.raises(AtfError) as e:
            sp.decode(idx, out=out)
        assert e.value.status == -8
        assert (out[:, 1] == -(2 ** 63)).all()
        with pytest.raises(AtfError) as e:
            sp.encode(torch.zeros((5, 2), dtype=torch.int32, device="cuda"))
        assert e.value.status == -10
    c1 = A.c1_toy()
    with GSpace(c1) as sp:
        sp.generate()
        idx = torch.arange(sp.size(), dtype=torch.int64, device="cuda")
        a = sp.decode(idx)
        b = sp.decode(idx, out=torch.empty((2, sp.size()), dtype=torch.int64, device="cuda"))
        assert a.dtype == torch.int32 and torch.equal(a.to(torch.int64), b)
