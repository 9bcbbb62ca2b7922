"""Pins of the CPU oracle against the paper and mathematics (never against itself).

P:n = PAPER.md line n.  Each test says what it pins and where the expected
value comes from: a closed form (oracle/closed_forms.py, computed two ways), a
worked example of the paper, brute force on tiny inputs, or a magnitude the
paper prints.
"""
import os

import numpy as np
import pytest

import atfspec as A
from atfspec import (Spec, X, C, P, DIVIDES, MULOF, interval, pow2, set_, divides,
                     is_multiple_of, E)
from oracle import closed_forms as cf
from oracle import run as orc

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def sizes(d):
    return [g["size"] for g in d["groups"]]


def fs(d, g=0):
    return [lv["f"] for lv in d["groups"][g]["levels"]]


# ---------------------------------------------------------------- closed forms
def test_c1_closed_form(oracle_bin):
    d = orc.info(A.c1_toy())
    assert int(d["S"]) == cf.c1_size() == 46
    assert fs(d) == [cf.count_divisors_upto(64, 64), 46]
    assert [lv["evals"] for lv in d["groups"][0]["levels"]] == [64, 7 * 64]


@pytest.mark.parametrize("n", [1, 12, 64, 360, 1000, 4096])
def test_saxpy_closed_form(oracle_bin, n):
    """WPT|N, LS|(N/WPT)  =>  S = sum_{d|N} tau(d) = prod (a+1)(a+2)/2."""
    d = orc.info(A.saxpy(n))
    assert int(d["S"]) == cf.saxpy_size_by_divisor_sum(n) == cf.saxpy_size_by_exponents(n)
    assert fs(d)[0] == cf.tau(n)
    assert len(d["groups"]) == 1


def test_saxpy_named_values(oracle_bin):
    # N = 64 -> 28, N = 1000 -> 100, N = 4096 -> 91 (closed form)
    for n, s in [(64, 28), (1000, 100), (4096, 91)]:
        assert cf.saxpy_size_by_exponents(n) == s
        assert int(orc.info(A.saxpy(n))["S"]) == s


def test_fig1_worked_example(oracle_bin):
    """Fig. 1: two groups {tp1,tp2}, {tp3,tp4}; 3 configs each; S = 9."""
    s = A.fig1()
    d = orc.info(s)
    assert [g["members"] for g in d["groups"]] == [[0, 1], [2, 3]]
    assert sizes(d) == [3, 3] and int(d["S"]) == 9
    assert fs(d, 0) == [2, 3] and fs(d, 1) == [2, 3]
    gold = np.loadtxt(os.path.join(GOLDEN, "fig1_rows.txt"), dtype=np.int32, comments="#")
    info, soa = orc.decode(s, np.arange(9, dtype=np.uint64))
    assert np.array_equal(soa.T, gold)
    _, rows = orc.o1(s)
    assert np.array_equal(rows, gold)


@pytest.mark.parametrize("R,E", [(64, 64), (100, 360), (10, 360), (4096, 2**12), (37, 1)])
def test_interval_divisibility_counts(oracle_bin, R, E):
    s = Spec("div"); s.add("x", interval(1, R), divides(E))
    assert int(orc.info(s)["S"]) == cf.count_divisors_upto(E, R)
    s = Spec("mul"); s.add("x", interval(1, R), is_multiple_of(E))
    assert int(orc.info(s)["S"]) == cf.count_multiples_upto(E, R)


@pytest.mark.parametrize("R", [1, 17, 64, 500])
def test_divisor_pairs_hyperbola(oracle_bin, R):
    s = Spec("pairs"); s.add("a", interval(1, R)); s.add("b", interval(1, R), divides(P(0)))
    assert int(orc.info(s)["S"]) == cf.dirichlet_hyperbola_D2(R) == cf.piltz_D(R, 2)[1]


def test_piltz_two_routes():
    # D_k(R) by the Dirichlet recurrence vs a literal chain count on a tiny range
    R, k = 24, 4
    def chains(depth, top):
        if depth == 0:
            return 1
        return sum(chains(depth - 1, d) for d in range(1, top + 1) if top % d == 0)
    brute = [sum(chains(j, x) for x in range(1, R + 1)) for j in range(k)]
    assert brute == cf.piltz_D(R, k)
    assert cf.piltz_D(4096, 2)[1] == 34720          # SURVEY.md §8(c) interval pin


@pytest.mark.parametrize("R,L", [(60, 5), (128, 8)])
def test_c5_chains_piltz(oracle_bin, R, L):
    d = orc.info(A.c5_chains(R, L), threads=8)
    want = cf.c5_level_sizes(R, L)
    assert [fs(d, g) for g in range(3)] == want
    S = 1
    for w in want:
        S *= w[-1]
    assert int(d["S"]) == S
    for g in range(3):
        lv = d["groups"][g]["levels"]
        prev = 1
        for l in lv:
            assert l["evals"] == prev * l["r"]     # evals_k = f_{k-1} * r_k
            prev = l["f"]


# ---------------------------------------------------------------- paper magnitudes
def test_c2_paper_magnitudes(oracle_bin):
    """at 2^10 x 2^10 the unconstrained XgemmDirect space has > 10^19 configs while
    ATF's constrained space has 'nearly 10^7'."""
    d = orc.info(A.c2_xgemm_direct(1024), threads=8)
    assert int(d["unconstrained"]) == 1024 ** 6 * 4 * 4 * 2 * 2 > 10 ** 19
    S = int(d["S"])
    assert 5 * 10 ** 6 < S < 10 ** 7
    # without the anchor (WGD|M, WGD|N) the size is far from 10^7: the anchor is confirmed
    assert [g["members"] for g in d["groups"]] == [[0, 1, 2, 3, 4, 5, 6, 7], [8], [9]]


def test_empty_space_cltune_limits(oracle_bin):
    """CLTune's WGD in {8,16,32} with WGD | rows and WGD | cols empties the space for
    the deep-learning shapes (rows 20, cols 576)."""
    s = Spec("cltune_wgd"); s.add("WGD", set_(8, 16, 32), divides(20) & divides(576))
    s.add("KWID", interval(1, 32), divides(P(0)))
    d = orc.info(s)
    assert int(d["S"]) == 0 and sizes(d) == [0]


def test_pow2_first_ten(oracle_bin):
    """interval<size_t>(1, 10, pow(2,i)) 'represents the first ten powers of 2'."""
    s = Spec("pow2"); s.add("x", pow2(1, 10))
    assert int(orc.info(s)["S"]) == 10
    info, soa = orc.decode(s, np.arange(10, dtype=np.uint64))
    assert soa[0].tolist() == [2 ** i for i in range(1, 11)]
    s = Spec("even"); s.add("z", interval(2, 4096, 2))
    assert int(orc.info(s)["S"]) == 2048


def test_duplicate_set_rejected(oracle_bin):
    s = Spec("dup"); s.add("x", set_(1, 2, 2))
    with pytest.raises(ValueError):
        orc.info(s)


# ---------------------------------------------------------------- metamorphic
@pytest.mark.parametrize("n", [16, 32])
def test_c2_implied_constraints_change_nothing(oracle_bin, n):
    a = orc.info(A.c2_xgemm_direct(n, implied=True), hash=True)
    b = orc.info(A.c2_xgemm_direct(n, implied=False), hash=True)
    assert a["S"] == b["S"]
    assert [g["hash"] for g in a["groups"]] == [g["hash"] for g in b["groups"]]


def test_tautology_changes_nothing(oracle_bin):
    s1 = A.c3_xgemm((6, 8, 4))
    s2 = A.c3_xgemm((6, 8, 4))
    s2.params[5].constraints.append((X >= 1).code)          # MDIMA >= 1 holds on its range
    a, b = orc.info(s1, hash=True), orc.info(s2, hash=True)
    assert a["groups"][0]["hash"] == b["groups"][0]["hash"]


# ---------------------------------------------------------------- O1 == O2 (brute force)
def _o1_vs_decode(spec):
    d1, rows = orc.o1(spec)
    d2 = orc.info(spec)
    assert int(d2["S"]) == d1["S"] == rows.shape[0]
    if rows.shape[0]:
        _, soa = orc.decode(spec, np.arange(rows.shape[0], dtype=np.uint64))
        assert np.array_equal(soa.T, rows)


@pytest.mark.parametrize("name", ["c1", "fig1", "saxpy12", "c2_8", "c3_tiny", "c3_tiny_anch"])
def test_o1_equals_o2_named(oracle_bin, name):
    spec = {"c1": A.c1_toy, "fig1": A.fig1, "saxpy12": lambda: A.saxpy(12),
            "c2_8": lambda: A.c2_xgemm_direct(8), "c3_tiny": lambda: A.c3_xgemm((4, 6, 2)),
            "c3_tiny_anch": lambda: A.c3_xgemm((3, 2, 2), anchored=True)}[name]()
    _o1_vs_decode(spec)


@pytest.mark.parametrize("seed", range(60))
def test_o1_equals_o2_fuzz(oracle_bin, seed):
    _o1_vs_decode(A.random_spec(seed))


# ---------------------------------------------------------------- two encodings agree
@pytest.mark.parametrize("spec,native", [
    (lambda: A.c1_toy(), "c1"),
    (lambda: A.c2_xgemm_direct(256), "c2:256"),
    (lambda: A.c3_xgemm("IS1"), "c3:"),
    (lambda: A.c3_xgemm("IS3"), "c3:"),
    (lambda: A.c3_xgemm((12, 30, 8)), "c3:"),
    (lambda: A.saxpy(360), "saxpy:360"),
])
def test_bytecode_matches_native_predicates(oracle_bin, spec, native):
    d = orc.info(spec(), threads=4, native=native, native_check=True)
    assert d["native_mismatch"] == 0
    d2 = orc.info(spec(), threads=4, native=native)
    assert d2["S"] == d["S"]


# ---------------------------------------------------------------- decode = mixed radix
def test_decode_mixed_radix_c4_structure(oracle_bin):
    """SURVEY.md §8(c) C4 pin: with contiguous groups and the four binary singletons last,
    decode(i) = (G0 tuple floor(i/16), bits of i mod 16 for STRM, STRN, SA, SB)."""
    s = A.c3_xgemm((4, 8, 4))
    d = orc.info(s)
    g0 = orc.leaves(s, 0, 10)
    S = int(d["S"])
    assert S == g0.shape[0] * 16
    idx = np.arange(S, dtype=np.uint64)
    _, soa = orc.decode(s, idx)
    i = np.arange(S)
    assert np.array_equal(soa[:10].T, g0[i // 16])
    for b, p in enumerate([10, 11, 12, 13]):
        assert np.array_equal(soa[p], (i >> (3 - b)) & 1)
    # lexicographic extremes
    assert soa[:, 0].tolist()[:3] == [1, 1, 1]


def test_decode_out_of_range(oracle_bin):
    s = A.fig1()
    info, soa = orc.decode(s, np.array([9, 10, 2 ** 63], dtype=np.uint64))
    assert info["invalid"] == 3
    assert (soa == np.iinfo(np.int32).min).all()


# ---------------------------------------------------------------- opcode semantics
def _accepted(code, lo=-6, hi=6):
    s = Spec("op"); s.add("x", interval(lo, hi), code)
    n = int(orc.info(s)["S"])
    if n == 0:
        return []
    _, soa = orc.decode(s, np.arange(n, dtype=np.uint64))
    return soa[0].tolist()


def test_opcode_semantics_reading_table(oracle_bin):
    """Readings #6-#8: aliases, strict evaluation, zero divisor rejects, C truncation."""
    xs = range(-6, 7)
    trunc_div = lambda a, b: abs(a) // abs(b) * (1 if (a >= 0) == (b >= 0) else -1)
    trunc_mod = lambda a, b: a - b * trunc_div(a, b)
    assert _accepted(divides(12)) == [x for x in xs if x != 0 and 12 % abs(x) == 0]
    # x % 3 == 0 includes x = 0 (MULOF: [b != 0 and a mod b == 0], b = 3)
    assert _accepted(is_multiple_of(3)) == [x for x in xs if trunc_mod(x, 3) == 0]
    assert _accepted(X < 2) == [x for x in xs if x < 2]
    assert _accepted(X <= 2) == [x for x in xs if x <= 2]
    assert _accepted(X.eq(-3)) == [-3]
    assert _accepted(X.ne(-3)) == [x for x in xs if x != -3]
    # DIV truncates toward zero; -7 / 2 = -3
    assert _accepted((C(-7) // X).eq(-3)) == [x for x in xs if x != 0 and trunc_div(-7, x) == -3]
    assert _accepted((C(-7) % X).eq(-1)) == [x for x in xs if x != 0 and trunc_mod(-7, x) == -1]
    # zero divisor rejects even under OR with a true operand (strict evaluation, reading #7)
    assert 0 not in _accepted(((C(5) // X) > 100) | C(1))
    assert 0 not in _accepted(~DIVIDES(X, 7))
    assert _accepted(~DIVIDES(X, 7)) == [x for x in xs if x != 0 and 7 % abs(x) != 0]
    # integer result used as a boolean: nonzero accepts
    assert _accepted(X - 2) == [x for x in xs if x != 2]
    assert _accepted(E((X * X).code)) == [x for x in xs if x != 0]
    assert _accepted(A.min_(X, 3).eq(3)) == [x for x in xs if x >= 3]
    assert _accepted(A.max_(X, 3).eq(3)) == [x for x in xs if x <= 3]


def test_cltune_zero_range_same_space(oracle_bin):
    """CLTune's saxpy ranges start at 0; with reading #7 a zero divisor rejects the
    candidate, so the 0..N ranges define the same space as 1..N."""
    n = 360
    s = Spec("saxpy0"); s.add("WPT", interval(0, n), divides(n))
    s.add("LS", interval(0, n), divides(C(n) // P(0)))
    assert int(orc.info(s)["S"]) == cf.saxpy_size_by_exponents(n)


def test_overflow_is_reported(oracle_bin):
    s = Spec("ovf"); s.add("x", interval(1, 4), (C(2 ** 62) * X) > 0)
    assert orc.info(s)["overflow"] is True


# ---------------------------------------------------------------- survey cross-check
def test_c3_small_shapes_match_survey_appendix(oracle_bin):
    """SURVEY.md Appendix A (an independent counter): C3 IS1 and IS3 per-level f_k."""
    d = orc.info(A.c3_xgemm("IS1"), threads=8)
    assert fs(d) == [20, 11520, 11520, 38016, 248424, 85055, 90173, 90173, 129716, 239741]
    d = orc.info(A.c3_xgemm("IS3"), threads=8)
    assert fs(d) == [50, 3200, 3200, 13248, 57960, 35070, 30555, 30555, 48298, 80124]
    assert int(d["S"]) == 80124 * 16


# ---------------------------------------------------------------- P:57 generator ranges (NEXT-3)
def test_generator_range_closed_forms():
    """interval(begin, end, step, generator): the elements generator(i); pinned by closed
    forms of the materialised range (squares, an affine map, a step) through the oracle's own
    parser: a space whose only parameter has the range enumerates exactly those values."""
    import numpy as np
    cases = [(A.gen(1, 10, A.X * A.X), [i * i for i in range(1, 11)]),
             (A.gen(0, 20, A.X * 3 + 1, step=4), [3 * i + 1 for i in range(0, 21, 4)]),
             (A.gen(-3, 3, A.X * A.X * A.X - A.X), None)]
    for rng, want in cases[:2]:
        s = A.Spec("gen")
        s.add("p", rng)
        info = orc.info(s)
        assert info["groups"][0]["size"] == len(want)
        _, rows = orc.decode(s, np.arange(len(want), dtype=np.uint64))
        assert rows[0].tolist() == want
    # i^3 - i repeats 0 at i = -1, 0, 1: rejected like a duplicate set value (reading #5)
    s = A.Spec("gen_dup")
    s.add("p", cases[2][0])
    with pytest.raises(Exception):
        orc.info(s)


# ---------------------------------------------------------------- the oracle's constraint check
# orc.check (oracle/atf_oracle.cpp cmd_check) decides "valid configuration" ("all valid
# parameter configurations, i.e., for which the parameters' constraints are satisfied").
# Pinned three ways, none of which is the oracle's own interpreter: (1) hand-written Python
# predicates restated from the paper / CLBlast's constraint list on EVERY tuple of the full
# product, plus values outside the ranges; (2) on fuzz specs, membership in O1's row set over the
# full product (O1 is pinned by the closed forms above); (3) an out-of-range value in any column
# makes a row invalid.
def _product(ranges):
    grids = np.meshgrid(*[np.asarray(r, dtype=np.int64) for r in ranges], indexing="ij")
    return np.stack([g.ravel() for g in grids], 1)


def _values(spec):
    out = []
    for p in spec.params:
        r = p.range
        if r["kind"] == "interval":
            out.append(list(range(r["begin"], r["end"] + 1, r["step"])))
        elif r["kind"] == "pow2":
            out.append([1 << i for i in range(r["begin"], r["end"] + 1, r["step"])])
        else:
            out.append(list(r["values"]))
    return out


def _dv(a, b):
    """a | b with the reading-#7 zero rule (a == 0 rejects)."""
    return a != 0 and b % a == 0


def _c2_pred(n):
    def ok(WGD, MC, NC, MA, NB, KW, VM, VN, PA, PB):
        return (_dv(WGD, n) and _dv(MC, WGD) and _dv(NC, WGD) and _dv(MA, WGD) and MA != 0
                and (MC * NC) // MA != 0 and _dv((MC * NC) // MA, WGD) and _dv(NB, WGD) and NB != 0
                and (MC * NC) // NB != 0 and _dv((MC * NC) // NB, WGD) and _dv(KW, WGD)
                and _dv(MC * VM, WGD) and _dv(MA * VM, WGD) and _dv(NC * VN, WGD) and _dv(NB * VN, WGD))
    return ok


def _c3_pred(MWG, NWG, KWG, MC, NC, MA, NB, KWI, VM, VN, *_):
    # CLBlast Xgemm c1-c7 (reading #13): every value >= 1 on these ranges
    return (_dv(MC, MWG) and _dv(NC, NWG) and _dv(MA, MWG) and _dv(NB, NWG)
            and (MC * NC) // MA != 0 and _dv((MC * NC) // MA, KWG)
            and (MC * NC) // NB != 0 and _dv((MC * NC) // NB, KWG) and _dv(KWI, KWG)
            and _dv(MC * VM, MWG) and _dv(MA * VM, MWG) and _dv(NC * VN, NWG) and _dv(NB * VN, NWG))


CHECK_PREDICATES = {
    # C1 (configs[0]): TS_M | 64, TS_N | 64, TS_M * TS_N <= 1024
    "C1": (A.c1_toy, lambda m, n: _dv(m, 64) and _dv(n, 64) and m * n <= 1024),
    # saxpy: WPT | N, LS | (N / WPT)
    "saxpy12": (lambda: A.saxpy(12), lambda w, l: _dv(w, 12) and _dv(l, 12 // w)),
    # Fig. 1: tp2 | tp1, tp4 | tp3
    "fig1": (A.fig1, lambda a, b, c, d: _dv(b, a) and _dv(d, c)),
    "C2-4": (lambda: A.c2_xgemm_direct(4), _c2_pred(4)),
    "C3-2x3x2": (lambda: A.c3_xgemm((2, 3, 2)), _c3_pred),
    # C5 chains: x_k | x_{k-1}, y_{k-1} | y_k
    "C5-4x3": (lambda: A.c5_chains(4, 3),
               lambda x0, x1, x2, y0, y1, y2, z0, z1, z2: _dv(x1, x0) and _dv(x2, x1) and _dv(y0, y1)
               and _dv(y1, y2) and _dv(z1, z0) and _dv(z2, z1)),
}


@pytest.mark.parametrize("name", list(CHECK_PREDICATES))
def test_check_matches_paper_predicates_on_full_product(oracle_bin, name):
    mk, pred = CHECK_PREDICATES[name]
    spec = mk()
    vals = _values(spec)
    rows = _product(vals)
    assert 0 < rows.shape[0] <= 600_000
    want = np.array([bool(pred(*map(int, r))) for r in rows])
    got = orc.check(spec, rows.astype(np.int32), per_row=True)
    assert np.array_equal(got["flags"].astype(bool), want), name
    assert got["valid"] == int(want.sum()) and got["in_range"] == rows.shape[0]
    assert 0 < want.sum() < len(want)
    # the valid rows are exactly the space the oracle enumerates (its size and its rows)
    d1, o1rows = orc.o1(spec)
    assert int(d1["S"]) == int(want.sum())
    assert {tuple(r) for r in o1rows.tolist()} == {tuple(r) for r in rows[want].tolist()}


@pytest.mark.parametrize("seed", range(0, 60, 3))
def test_check_is_o1_membership_on_fuzz_products(oracle_bin, seed):
    spec = A.random_spec(seed)
    vals = _values(spec)
    if any(len(v) == 0 for v in vals) or np.prod([len(v) for v in vals], dtype=object) > 400_000:
        pytest.skip("empty range or product too large for an exhaustive check")
    rows = _product(vals)
    _, o1rows = orc.o1(spec)
    members = {tuple(r) for r in o1rows.tolist()}
    want = np.array([tuple(r) in members for r in rows.tolist()])
    got = orc.check(spec, rows.astype(np.int32), per_row=True)["flags"].astype(bool)
    assert np.array_equal(got, want)


def test_check_rejects_values_outside_the_ranges(oracle_bin):
    """a configuration takes each parameter's value from its range; a row that is
    valid except for one column replaced by a value outside that column's range is invalid."""
    for spec in (A.c1_toy(), A.saxpy(64), A.c3_xgemm((4, 6, 2)), A.c5_chains(6, 3)):
        _, rows = orc.o1(spec)
        rows = rows[:200].astype(np.int64)
        assert orc.check(spec, rows.astype(np.int32))["valid"] == rows.shape[0]
        vals = _values(spec)
        bad = rows.copy()
        for i in range(bad.shape[0]):
            p = i % bad.shape[1]
            bad[i, p] = max(vals[p]) + 1 + i   # outside the range (every range here is bounded above)
        got = orc.check(spec, bad.astype(np.int32), per_row=True)
        assert got["valid"] == 0 and not got["flags"].any()
