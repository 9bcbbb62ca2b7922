"""GPU parity: the CUDA path (through the C ABI) vs the CPU oracle, bit-exact.

Integer work throughout: sizes (u128), per-level node counts f_k, every decoded
configuration (small spaces, all indices) and order-dependent hashes of whole
groups / sampled decodes at full size (goldens written by tests/golden/make_golden.py,
which calls only oracle/).  Every input is a deterministic spec from atfspec or a
seeded fuzz spec.
"""
import json
import os

import numpy as np
import pytest

import atfspec as A
from atfspec.fuzz import splitmix64_indices
from oracle import closed_forms as cf
from oracle import run as orc

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


@pytest.fixture(scope="module")
def Space():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_hpdc_raschg18_b200 import Space as S
    return S


def _flags(generic):
    from paper_conf_hpdc_raschg18_b200 import _lib as L
    return L.ATF_FLAG_GENERIC_ONLY if generic else 0


def torch_rowhash(rows_pm: "torch.Tensor", base: int = 0) -> int:
    """Same definition as the oracle's: H = sum_i rowhash(row_i) * (2 (base+i) + 1) mod 2^64.
    rows_pm: int32 [P, n] (SoA), computed on the GPU with wrapping int64 arithmetic."""
    P, n = rows_pm.shape
    M32 = 0xFFFFFFFF
    z = torch.full((n,), 0x243F6A8885A308D3, dtype=torch.int64, device=rows_pm.device)
    K = torch.tensor(0x9E3779B97F4A7C15 - (1 << 64), dtype=torch.int64, device=rows_pm.device)
    for p in range(P):
        z = z ^ (rows_pm[p].to(torch.int64) & M32)
        z = z * K
        z = z ^ ((z >> 32) & M32)
    w = torch.arange(base, base + n, dtype=torch.int64, device=rows_pm.device) * 2 + 1
    s = (z * w).sum()  # wraps mod 2^64
    return int(s.item()) & ((1 << 64) - 1)


def _check_against_oracle(Space, spec, generic=False, decode_all_max=3_000_000, legacy=False, no_jit=False,
                          extra_flags=0, leaves_max=4_000_000, regenerate=False):
    """Sizes, groups, f_k and evals vs the oracle; then CONTENT: every configuration (decode of
    all S indices) when S <= decode_all_max, else every group's leaves element by element
    (decode_digits over all of the group's leaves vs the oracle's canonical leaf stream) for
    groups of at most leaves_max leaves."""
    from paper_conf_hpdc_raschg18_b200 import _lib as L
    ref = orc.info(spec, threads=8)
    flags = (_flags(generic) | (L.ATF_FLAG_LEGACY_WIDE if legacy else 0) | (L.ATF_FLAG_NO_JIT if no_jit else 0)
             | extra_flags)
    with Space(spec, flags=flags) as sp:
        sp.generate()
        if regenerate:        # the second generation of a space replays the first one's level sizes;
            for _ in range(3):  # the third is captured as a CUDA graph, the fourth launches it
                sp.generate()
        assert sp.groups() == [g["members"] for g in ref["groups"]]
        assert sp.size() == int(ref["S"])
        assert sp.group_sizes() == [g["size"] for g in ref["groups"]]
        for g, grp in enumerate(ref["groups"]):
            assert sp.level_sizes(g) == [lv["f"] for lv in grp["levels"]], (spec.name, g)
        st = sp.stats()
        evals = [lv["evals"] for grp in ref["groups"] for lv in grp["levels"]]
        assert [x["evals"] for x in st] == evals
        S = sp.size()
        if 0 < S <= decode_all_max:
            idx = torch.arange(S, dtype=torch.int64, device="cuda")
            got = sp.decode(idx).cpu().numpy()
            _, want = orc.decode(spec, np.arange(S, dtype=np.uint64))
            assert np.array_equal(got, want), spec.name
        elif S > decode_all_max:
            checked = 0
            for g, grp in enumerate(ref["groups"]):
                if grp["size"] > leaves_max:
                    continue
                assert _group_leaves(sp, g, grp["size"]).equal(
                    torch.from_numpy(orc.leaves(spec, g, len(grp["members"])))), (spec.name, g)
                checked += 1
            assert checked, spec.name


def _group_leaves(sp, g, size, start=0, chunk=1 << 22):
    """Leaves [start, start+size) of group g as int32 [n][members] (host), via decode_digits."""
    members = sp.groups()[g]
    G = sp.num_groups()
    parts = []
    for s0 in range(start, start + size, chunk):
        n = min(chunk, start + size - s0)
        dig = torch.zeros((G, n), dtype=torch.int64, device="cuda")
        dig[g] = torch.arange(s0, s0 + n, dtype=torch.int64, device="cuda")
        parts.append(sp.decode_digits(dig)[members].T.cpu())
    return torch.cat(parts) if parts else torch.zeros((0, len(members)), dtype=torch.int32)


SMALL = {
    "C1": A.c1_toy,
    "fig1": A.fig1,
    "saxpy64": lambda: A.saxpy(64),
    "saxpy360": lambda: A.saxpy(360),
    "saxpy1": lambda: A.saxpy(1),
    "C2-32": lambda: A.c2_xgemm_direct(32),
    "C2-256": lambda: A.c2_xgemm_direct(256),
    "C2-64-noimplied": lambda: A.c2_xgemm_direct(64, implied=False),
    "C3-12x30x8": lambda: A.c3_xgemm((12, 30, 8)),
    "C3-IS1": lambda: A.c3_xgemm("IS1"),
    "C3-IS3": lambda: A.c3_xgemm("IS3"),
    "C3-IS4-anch": lambda: A.c3_xgemm("IS4", anchored=True),
    "C5-60x5": lambda: A.c5_chains(60, 5),
    "C5-300x4": lambda: A.c5_chains(300, 4),
    # full-width ranges: nodes with 4096 children (y-chain value 1), heavy first tiles
    "C5-4096x3": lambda: A.c5_chains(4096, 3),
}


@pytest.mark.parametrize("name", list(SMALL))
@pytest.mark.parametrize("generic", [False, True])
def test_small_specs(Space, name, generic):
    _check_against_oracle(Space, SMALL[name](), generic=generic)


@pytest.mark.parametrize("name", list(SMALL))
def test_small_specs_regenerated(Space, name):
    """Steady state: later generations of a space (replay of the first one's level sizes, one
    synchronisation; from the third on one CUDA graph launch) give the same space, headline flags
    and default flags."""
    from paper_conf_hpdc_raschg18_b200 import _lib as L
    _check_against_oracle(Space, SMALL[name](), regenerate=True)
    _check_against_oracle(Space, SMALL[name](), regenerate=True, extra_flags=L.ATF_FLAG_NO_SEG_BOUNDS)


def test_graph_replay_follows_buffer_moves(Space):
    """The captured replay graph references the space's buffers: an operation that reallocates
    one between generations (here: decodes of growing size) makes the next generation capture a
    new graph; every generation's levels equal the first one's."""
    from paper_conf_hpdc_raschg18_b200 import _lib as L
    spec = A.c3_xgemm((20, 96, 8))
    with Space(spec, flags=L.ATF_FLAG_NO_SEG_BOUNDS) as sp:
        sp.generate()
        G = sp.num_groups()
        want = [[tuple(t.clone() if t is not None else None for t in sp.level_tensors(g, k))
                 for k in range(sp.num_levels(g))] for g in range(G)]
        S = sp.size()
        for i in range(6):
            if i in (3, 4):
                n = min(S, 1000 * (10 ** i))
                sp.decode(torch.arange(n, dtype=torch.int64, device="cuda") % S)
            sp.generate()
            for g in range(G):
                for k in range(sp.num_levels(g)):
                    rec, csr = sp.level_tensors(g, k)
                    assert torch.equal(rec, want[g][k][0]), (i, g, k)
                    if csr is not None:
                        assert torch.equal(csr, want[g][k][1]), (i, g, k)


@pytest.mark.parametrize("seed", range(0, 80, 3))
def test_fuzz_specs_regenerated(Space, seed):
    _check_against_oracle(Space, A.random_spec(seed), regenerate=True)
    _check_against_oracle(Space, A.random_wide_spec(seed % 40), regenerate=True)


@pytest.mark.parametrize("name", ["C5-60x5", "C5-300x4", "C5-4096x3", "C2-256", "C3-IS1", "C3-12x30x8"])
def test_small_specs_every_pair_evaluated(Space, name):
    """ATF_FLAG_NO_SEG_BOUNDS (the bench headline's configuration: all f_{k-1} r_k pairs
    evaluated) gives the same space."""
    from paper_conf_hpdc_raschg18_b200 import _lib as L
    _check_against_oracle(Space, SMALL[name](), extra_flags=L.ATF_FLAG_NO_SEG_BOUNDS)


@pytest.mark.parametrize("seed", range(80))
def test_fuzz_specs(Space, seed):
    _check_against_oracle(Space, A.random_spec(seed))


@pytest.mark.parametrize("seed", range(0, 80, 4))
def test_fuzz_specs_generic(Space, seed):
    _check_against_oracle(Space, A.random_spec(seed), generic=True)


@pytest.mark.parametrize("seed", range(40))
def test_fuzz_wide_specs(Space, seed):
    """Ranges of 65..6000 values (the wide kernel: hot filters x|n, d|x, (a x)|n, generic
    conjuncts, chunked ranges > 4096, zero and negative candidates) vs the oracle."""
    _check_against_oracle(Space, A.random_wide_spec(seed))


@pytest.mark.parametrize("seed", range(0, 40, 3))
def test_fuzz_wide_specs_legacy_kernel(Space, seed):
    """The block-tile wide kernel (ATF_FLAG_LEGACY_WIDE) on the same specs."""
    _check_against_oracle(Space, A.random_wide_spec(seed), legacy=True)


@pytest.mark.parametrize("name", ["C1", "C2-256", "C3-IS1", "C3-IS3", "C3-12x30x8", "saxpy360"])
def test_small_specs_generic_narrow_kernel(Space, name):
    """The generic (not NVRTC-specialised) narrow fast kernel on the same specs."""
    _check_against_oracle(Space, SMALL[name](), no_jit=True)


@pytest.mark.parametrize("seed", range(0, 80, 9))
def test_fuzz_specs_generic_narrow_kernel(Space, seed):
    _check_against_oracle(Space, A.random_spec(seed), no_jit=True)


@pytest.mark.parametrize("name", ["C1", "C2-256", "C3-IS1", "C3-IS3", "C3-12x30x8", "saxpy360", "C5-300x4"])
def test_small_specs_without_tail(Space, name):
    """ATF_FLAG_NO_TAIL: the trailing narrow levels one level at a time (expand_nfast +
    nfast_emit) instead of the fused tail give the same space."""
    from paper_conf_hpdc_raschg18_b200 import _lib as L
    _check_against_oracle(Space, SMALL[name](), extra_flags=L.ATF_FLAG_NO_TAIL)


@pytest.mark.parametrize("name", ["C2-256", "C3-IS1", "C3-12x30x8"])
def test_small_specs_generic_tail(Space, name):
    """The generic (not NVRTC-specialised) fused tail kernels."""
    from paper_conf_hpdc_raschg18_b200 import _lib as L
    _check_against_oracle(Space, SMALL[name](), no_jit=True)


@pytest.mark.parametrize("seed", range(0, 80, 7))
def test_fuzz_specs_without_tail(Space, seed):
    from paper_conf_hpdc_raschg18_b200 import _lib as L
    _check_against_oracle(Space, A.random_spec(seed), extra_flags=L.ATF_FLAG_NO_TAIL)


def test_tail_kernel_runs(Space):
    """C3's trailing narrow levels KWI, VWM, VWN (and C2's VWMD, VWND) run as one fused tail
    (kernel id 5 / 6).  Their terms read only ancestors above the tail, so the tail is
    product-structured: the first tail level evaluates every (frontier node, candidate) pair, a
    deeper level's mask is evaluated once per frontier node (stats "pairs" = f_frontier x r_d);
    with the product count off, every pair counts."""
    from paper_conf_hpdc_raschg18_b200 import _lib as L
    for spec, want in ((A.c3_xgemm("IS1"), [7, 8, 9]), (A.c2_xgemm_direct(256), [6, 7])):
        with Space(spec, flags=L.ATF_FLAG_TIMING) as sp:
            sp.generate()
            st = [x for x in sp.stats() if x["group"] == 0]
            assert [x["level"] for x in st if x["kernel"] == 6] == want   # NVRTC-specialised tail
            tail = [x for x in st if x["kernel"] == 6]
            f_front = st[want[0] - 1]["f"]
            assert tail[0]["pairs"] == tail[0]["evals"]
            assert all(x["pairs"] == f_front * x["r"] for x in tail[1:])
        L.check(L.atf_test_set_tail_product(0))
        try:
            with Space(spec, flags=L.ATF_FLAG_TIMING) as sp:
                sp.generate()
                st = [x for x in sp.stats() if x["group"] == 0]
                assert all(x["pairs"] == x["evals"] for x in st if x["kernel"] == 6)
        finally:
            L.check(L.atf_test_set_tail_product(1))
        with Space(spec, flags=L.ATF_FLAG_TIMING | L.ATF_FLAG_NO_JIT) as sp:
            sp.generate()
            assert [x["level"] for x in sp.stats() if x["group"] == 0 and x["kernel"] == 5] == want


def test_extended_tail_runs(Space):
    """C3-IS4: the NVRTC tail also takes KWI (r = 64 > 32, u64 masks) since its frontier (NDIMB's
    level, 6.8e6 nodes) is large; the generic tail kernels keep the r <= 32 run VWM, VWN.  Both
    generate the golden space (test_full_size_against_golden covers the content)."""
    from paper_conf_hpdc_raschg18_b200 import _lib as L
    spec = A.c3_xgemm("IS4")
    for flags, kern, want in ((0, 6, [7, 8, 9]), (L.ATF_FLAG_NO_JIT, 5, [8, 9])):
        with Space(spec, flags=L.ATF_FLAG_TIMING | flags) as sp:
            sp.generate()
            st = [x for x in sp.stats() if x["group"] == 0]
            assert [x["level"] for x in st if x["kernel"] == kern] == want
            assert sp.size() == 1613777840


def test_jit_kernels_run(Space):
    """The narrow levels of C3 run the NVRTC-specialised kernel (kernel id 4) on the GPU box."""
    from paper_conf_hpdc_raschg18_b200 import _lib as L
    with Space(A.c3_xgemm("IS1"), flags=L.ATF_FLAG_TIMING) as sp:
        sp.generate()
        kinds = [st["kernel"] for st in sp.stats()]
        assert 4 in kinds, kinds


@pytest.mark.parametrize("name", ["C3-IS1", "C5-300x4", "C5-4096x3", "C2-256"])
def test_small_specs_legacy_kernel(Space, name):
    _check_against_oracle(Space, SMALL[name](), legacy=True)


@pytest.mark.parametrize("seed", range(0, 40, 5))
def test_fuzz_wide_specs_generic(Space, seed):
    _check_against_oracle(Space, A.random_wide_spec(seed), generic=True)


def test_wide_ranges_chunked(Space):
    """r > 4096 candidates per level -> several candidate chunks per frontier node."""
    _check_against_oracle(Space, A.saxpy(5040 * 4))
    s = A.Spec("wide")
    s.add("a", A.interval(1, 12))
    s.add("b", A.interval(1, 20000), A.divides(A.P(0) * 1000) | (A.X > 19990))
    _check_against_oracle(Space, s)


def test_empty_space(Space):
    s = A.Spec("cltune_wgd")
    s.add("WGD", A.set_(8, 16, 32), A.divides(20) & A.divides(576))
    s.add("KWID", A.interval(1, 32), A.divides(A.P(0)))
    with Space(s) as sp:
        sp.generate()
        assert sp.size() == 0 and sp.level_sizes(0) == [0, 0]
        from paper_conf_hpdc_raschg18_b200 import AtfError
        with pytest.raises(AtfError):
            sp.decode(torch.zeros(3, dtype=torch.int64, device="cuda"))


def test_decode_out_of_range_rows(Space):
    from paper_conf_hpdc_raschg18_b200 import AtfError
    with Space(A.fig1()) as sp:
        sp.generate()
        idx = torch.tensor([0, 8, 9, 1 << 40], dtype=torch.int64, device="cuda")
        out = torch.empty((4, 4), dtype=torch.int32, device="cuda")
        with pytest.raises(AtfError) as e:
            sp.decode(idx, out=out)
        assert e.value.status == -8
        o = out.cpu().numpy()
        assert (o[:, 2:] == np.iinfo(np.int32).min).all()
        assert o[:, 0].tolist() == [1, 1, 1, 1] and o[:, 1].tolist() == [2, 2, 2, 2]


def test_csr_and_records_consistent(Space):
    spec = A.c3_xgemm((12, 30, 8))
    with Space(spec) as sp:
        sp.generate()
        L = sp.num_levels(0)
        pj = sp.plan_json()["groups"][0]["levels"]
        for k in range(L - 1):
            rec, csr = sp.level_tensors(0, k)
            crec, _ = sp.level_tensors(0, k + 1)
            csr = csr.cpu().numpy()
            assert csr[0] == 0 and csr[-1] == crec.shape[0] and (np.diff(csr) >= 0).all()
            # every child carries its parent's path plus one new field (level k+1)
            parent_of = np.repeat(np.arange(rec.shape[0]), np.diff(csr))
            r, c = rec.cpu().numpy().astype(np.int64), crec.cpu().numpy().astype(np.int64)
            w, sh, b = pj[k + 1]["word"], pj[k + 1]["shift"], pj[k + 1]["bits"]
            mask = ((1 << b) - 1) << sh
            c_wo = c.copy()
            c_wo[:, w] &= ~mask & 0xFFFFFFFF
            r_u = r & 0xFFFFFFFF
            assert np.array_equal(c_wo & 0xFFFFFFFF, r_u[parent_of])
            # children of one parent have strictly increasing range positions
            pos = (c[:, w] & 0xFFFFFFFF) >> sh & ((1 << b) - 1)
            same = parent_of[1:] == parent_of[:-1]
            assert (pos[1:][same] > pos[:-1][same]).all()


@pytest.mark.parametrize("n", [0, 1, 31, 1024, 1025, 1 << 20, 3_000_001])
def test_lookback_scan(Space, n):
    from paper_conf_hpdc_raschg18_b200 import _lib as L
    g = torch.Generator().manual_seed(n)
    for kind in ("rand", "zeros", "max", "one_huge"):
        if kind == "rand":
            x = torch.randint(0, 1000, (n,), generator=g, dtype=torch.int64)
        elif kind == "zeros":
            x = torch.zeros(n, dtype=torch.int64)
        elif kind == "max":
            x = torch.full((n,), 0xFFFFFFFF, dtype=torch.int64)
        else:
            x = torch.zeros(n, dtype=torch.int64)
            if n:
                x[n // 2] = 0xFFFFFFFF
        d_in = x.to(torch.int32).cuda() if n else torch.zeros(1, dtype=torch.int32, device="cuda")
        d_out = torch.empty(n + 1, dtype=torch.int64, device="cuda")
        L.check(L.atf_test_exclusive_scan_u32(d_in.data_ptr(), d_out.data_ptr(), n, None))
        want = np.concatenate([np.zeros(1, np.uint64), np.cumsum(x.numpy().astype(np.uint64))])  # exact u64 (no float64 promotion)
        assert np.array_equal(d_out.cpu().numpy().view(np.uint64), want), kind


# ---------------------------------------------------------------- full sizes (goldens)
def _golden(name):
    with open(os.path.join(GOLDEN, f"{name}.json")) as f:
        return json.load(f)


def _group_hash(sp, g, size, n_params, chunk=1 << 24):
    """Hash of group g's leaves (values of its members) in canonical order, via decode_digits."""
    G = sp.num_groups()
    members = sp.groups()[g]
    H = 0
    for s0 in range(0, size, chunk):
        n = min(chunk, size - s0)
        dig = torch.zeros((G, n), dtype=torch.int64, device="cuda")
        dig[g] = torch.arange(s0, s0 + n, dtype=torch.int64, device="cuda")
        out = sp.decode_digits(dig)
        H = (H + torch_rowhash(out[members], base=s0)) & ((1 << 64) - 1)
        del out, dig
    return H


FULL = ["C2", "C2-1024", "C3-IS1", "C3-IS3", "C3-IS2", "C3-IS4", "C3-IS4-anchored", "C5-512", "C5"]


@pytest.mark.parametrize("every_pair", [True, False])
@pytest.mark.parametrize("name", FULL)
def test_full_size_against_golden(Space, name, every_pair):
    """Full-size configs (C5 = configs[4] at 4096 x 8, the bench workload) in both launch
    configurations bench.py times (every pair evaluated = the headline; segment bounds = the
    secondary line): S, every f_k, the order-dependent hash of every group's leaves (all of
    them, in canonical order), element-wise windows of leaf rows (first / middle / last 1024
    leaves of every group, where the golden has them) and the C4 sampled decodes."""
    from paper_conf_hpdc_raschg18_b200 import _lib as L
    from tests.golden.make_golden import SPECS
    gold = _golden(name)
    spec = SPECS[name]()
    with Space(spec, flags=L.ATF_FLAG_NO_SEG_BOUNDS if every_pair else 0) as sp:
        sp.generate()
        sp.generate()   # the bench's timed steps: the second generation replays the level sizes
        assert sp.size() == int(gold["S"])
        for g, grp in enumerate(gold["groups"]):
            assert sp.level_sizes(g) == [lv["f"] for lv in grp["levels"]]
            assert _group_hash(sp, g, grp["size"], len(spec.params)) == int(grp["hash"]), (name, g)
        for g, wins in enumerate(gold.get("windows", [])):
            for w in wins:
                want = torch.tensor(w["rows"], dtype=torch.int32)
                got = _group_leaves(sp, g, want.shape[0], start=w["start"])
                assert got.equal(want), (name, g, w["start"])
        if "decode" in gold:
            d = gold["decode"]
            idx = torch.from_numpy(splitmix64_indices(d["n"], int(gold["S"]), d["seed"]).view(np.int64)).cuda()
            out = sp.decode(idx)
            assert torch_rowhash(out) == int(d["hash"])
            assert out[:, :8].T.cpu().tolist() == d["first_rows"]


def test_c4_decode_all_1e8_indices(Space):
    """configs[3] in full: decode of all 10^8 splitmix indices into C3-IS2 (the bench's C4
    launch: one decode_indices call over the whole batch), compared with the oracle's hash of
    all 10^8 rows (tests/golden/C3-IS2.json "decode_full"), plus 2*10^6 rows element by element
    against the oracle's own decode (a window at the start and one at the end of the batch)."""
    from tests.golden.make_golden import SPECS
    gold = _golden("C3-IS2")
    d = gold["decode_full"]
    spec = SPECS["C3-IS2"]()
    S = int(gold["S"])
    idx_h = splitmix64_indices(d["n"], S, d["seed"])
    with Space(spec) as sp:
        sp.generate()
        idx = torch.from_numpy(idx_h.view(np.int64)).cuda()
        out = sp.decode(idx)                       # [14][10^8] int32, 5.6 GB
        del idx
        H, chunk = 0, 1 << 24
        for s0 in range(0, d["n"], chunk):
            H = (H + torch_rowhash(out[:, s0:s0 + chunk], base=s0)) & ((1 << 64) - 1)
        assert H == int(d["hash"])
        for s0 in (0, d["n"] - 1_000_000):
            sel = idx_h[s0:s0 + 1_000_000]
            _, want = orc.decode(spec, sel, threads=8)
            assert np.array_equal(out[:, s0:s0 + 1_000_000].cpu().numpy(), want), s0


def test_c5_full_closed_form(Space):
    """C5 at full size (configs[4]): f_k = D_k(4096) for the x/y chains and D_k(2048) for z
    (Piltz; oracle/closed_forms.py), S = product of the leaf levels (u128)."""
    spec = A.c5_chains(4096, 8)
    want = cf.c5_level_sizes(4096, 8)
    with Space(spec) as sp:
        sp.generate()
        assert [sp.level_sizes(g) for g in range(3)] == want
        assert sp.size() == want[0][-1] * want[1][-1] * want[2][-1]
        # sampled decode: rows are valid configurations (checked by the oracle's constraint test)
        dig = torch.stack([torch.randint(0, want[g][-1], (4096,), device="cuda") for g in range(3)])
        rows = sp.decode_digits(dig).T.contiguous().cpu().numpy()
        chk = orc.check(spec, rows)
        assert chk["valid"] == chk["rows"] == 4096
        # lexicographic extremes: digit 0 = the first valid tuple in range-position order
        first = sp.decode_digits(torch.zeros((3, 1), dtype=torch.int64, device="cuda")).flatten().tolist()
        assert first == [1] * 16 + [2] * 8


# ---------------------------------------------------------------- encode (inverse decode)
def _range_values(r):
    """Range of a parameter as written in the spec: INTERVAL inclusive, POW2 = 2^i, SET listed."""
    if r["kind"] == "interval":
        return list(range(r["begin"], r["end"] + 1, r["step"]))
    if r["kind"] == "pow2":
        return [1 << i for i in range(r["begin"], r["end"] + 1, r["step"])]
    return list(r["values"])


def _perturb(spec, rows, gen):
    """Each row with one parameter replaced by a random value of its range (or a value
    outside every range): a mix of rows inside and outside the space."""
    rows = rows.copy()
    n, P = rows.shape
    ranges = [np.array(_range_values(p.range), dtype=np.int64) for p in spec.params]
    which = gen.integers(0, P, n)
    for i in range(n):
        R = ranges[which[i]]
        rows[i, which[i]] = R[gen.integers(0, len(R))] if gen.random() < 0.85 else 1_000_003
    return rows


@pytest.mark.parametrize("name", ["C1", "fig1", "saxpy360", "C2-256", "C3-IS1", "C3-12x30x8", "C5-300x4",
                                  "C3-IS4-anch"])
def test_encode_inverts_decode_and_tests_membership(Space, name):
    spec = SMALL[name]()
    gen = np.random.default_rng(7)
    with Space(spec) as sp:
        sp.generate()
        S = sp.size()
        if S < (1 << 63):
            n = min(S, 100_000)
            idx = torch.from_numpy(gen.integers(0, S, n, dtype=np.int64)).cuda() if S > n else \
                torch.arange(S, dtype=torch.int64, device="cuda")
            rows = sp.decode(idx)
            assert torch.equal(sp.encode(rows), idx)
        else:
            G = sp.num_groups()
            sizes = sp.group_sizes()
            n = 100_000
            dig = torch.stack([torch.from_numpy(gen.integers(0, sizes[g], n, dtype=np.int64)) for g in range(G)]).cuda()
            rows = sp.decode_digits(dig)
            assert torch.equal(sp.encode_digits(rows), dig)
        # membership of perturbed rows == the oracle's constraint check
        pert = _perturb(spec, rows.T.cpu().numpy(), gen)[:20_000]
        got = sp.encode_digits(torch.from_numpy(pert.T.copy()).cuda())
        got_valid = (got >= 0).all(dim=0).cpu().numpy()
        want = orc.check(spec, pert, per_row=True)["flags"].astype(bool)
        assert np.array_equal(got_valid, want)
        assert 0 < want.sum() < len(want) or S == 0


@pytest.mark.parametrize("seed", range(0, 80, 8))
def test_encode_fuzz_membership(Space, seed):
    spec = A.random_spec(seed)
    gen = np.random.default_rng(seed)
    with Space(spec) as sp:
        sp.generate()
        S = sp.size()
        ranges = [np.array(_range_values(p.range), dtype=np.int64) for p in spec.params]
        n = 5000
        rows = np.stack([R[gen.integers(0, len(R), n)] if len(R) else np.zeros(n, np.int64) for R in ranges], 1)
        got = sp.encode_digits(torch.from_numpy(rows.T.astype(np.int32).copy()).cuda())
        got_valid = (got >= 0).all(dim=0).cpu().numpy()
        want = orc.check(spec, rows.astype(np.int32), per_row=True)["flags"].astype(bool)
        assert np.array_equal(got_valid, want)
        if S and S < (1 << 63):
            idx = torch.arange(min(S, 4096), dtype=torch.int64, device="cuda")
            assert torch.equal(sp.encode(sp.decode(idx)), idx)


# ---------------------------------------------------------------- CLTune-style full-product filter
@pytest.mark.parametrize("name", ["C1", "fig1", "saxpy360", "C2-8", "C3-4x5x3", "C3-3x4x2-anch"])
def test_filter_product_counts_the_space(Space, name):
    """filtering the full product yields the same set as ATF's constrained ranges;
    here its size, against the oracle's O1 (literal brute force) and the tree generator."""
    spec = {"C1": A.c1_toy, "fig1": A.fig1, "saxpy360": lambda: A.saxpy(360),
            "C2-8": lambda: A.c2_xgemm_direct(8), "C3-4x5x3": lambda: A.c3_xgemm((4, 5, 3)),
            "C3-3x4x2-anch": lambda: A.c3_xgemm((3, 4, 2), anchored=True)}[name]()
    with Space(spec) as sp:
        cnt, tot = sp.filter_product()
        sp.generate()
        assert cnt == sp.size()
    o1, _ = orc.o1(spec)
    assert cnt == int(o1["S"])
    assert tot == int(np.prod([len(_range_values(p.range)) for p in spec.params], dtype=object))


@pytest.mark.parametrize("seed", range(0, 80, 5))
def test_filter_product_fuzz(Space, seed):
    spec = A.random_spec(seed)
    with Space(spec) as sp:
        cnt, _ = sp.filter_product()
        sp.generate()
        assert cnt == sp.size()


# ---------------------------------------------------------------- multi-GPU protocol, virtual ranks
@pytest.mark.parametrize("world", [2, 3, 8])
@pytest.mark.parametrize("name", ["C5-300x4", "C3-IS1", "C2-256", "C5-4096x3"])
def test_virtual_shards_concatenate_to_single_gpu(Space, world, name):
    """S§8(e) on one GPU: `world` spaces each expand their rank's slice (generate_shard), the
    counts are exchanged (here in-process instead of NCCL) and finalize_shard fixes global
    offsets.  Every rank reports the global group sizes, and the rank slices of every level,
    in rank order, are the single-GPU arrays bit for bit."""
    spec = SMALL[name]()
    with Space(spec) as one:
        one.generate()
        G = one.num_groups()
        ref = {(g, k): one.level_tensors(g, k)[0].clone() for g in range(G) for k in range(one.num_levels(g))}
        sizes = one.group_sizes()
    shards = [Space(spec) for _ in range(world)]
    try:
        counts = [sp.generate_shard(r, world) for r, sp in enumerate(shards)]
        for sp in shards:
            sp.finalize_shard(counts)
        for sp in shards:
            assert sp.group_sizes() == sizes
        for (g, k), want in ref.items():
            parts = []
            for sp in shards:
                v = sp.level_view(g, k)
                rec, _ = sp.level_tensors(g, k)
                parts.append((v["offset"], rec))
            if all(off == 0 and rec.shape[0] == want.shape[0] for off, rec in parts):
                for _, rec in parts:          # replicated prefix level
                    assert torch.equal(rec, want)
                continue
            parts.sort(key=lambda t: t[0])
            pos = 0
            for off, rec in parts:
                assert off == pos, (g, k)
                pos += rec.shape[0]
            assert torch.equal(torch.cat([rec for _, rec in parts]), want), (g, k)
    finally:
        for sp in shards:
            sp.close()


def test_generator_ranges_against_oracle(Space):
    """P:57 generator ranges (NEXT-3): a GEMM-like space whose tile sizes are generated
    (squares, powers of two by doubling expression, an affine map) vs the oracle."""
    s = A.Spec("gen_space")
    s.add("T", A.gen(1, 24, A.X * A.X))                                        # 1, 4, ..., 576
    s.add("U", A.gen(0, 9, A.X * 64 + 1), A.divides(A.P(0) * 64 + 64) | (A.X < 100))
    s.add("V", A.gen(1, 40, A.X * 3, step=1), A.divides(A.P(0)))
    s.add("W", A.interval(1, 200), A.divides(A.P(2) * 4))
    _check_against_oracle(Space, s)
    _check_against_oracle(Space, s, generic=True)


def test_divisible16_exhaustive(Space):
    """q | nb through an fp32 reciprocal (16-bit quotient divisors) = integer modulo on all 2^32 pairs."""
    import ctypes as C
    from paper_conf_hpdc_raschg18_b200 import _lib as L
    bad = C.c_uint64(1)
    L.check(L.atf_test_divisible16(C.byref(bad)))
    assert bad.value == 0


def test_enum_parameters(Space):
    """Named enumerations (NEXT-3): SETs of codes in listed order; constraints compare codes;
    decode + to_named give the names; the space equals the oracle's."""
    s = A.Spec("enum_space")
    mem = A.enum("global", "local", "private")
    s.add("MEM", mem)
    s.add("TS", A.interval(1, 64), A.divides(64) & ((A.P(0).eq(A.enum_code(mem, "local"))) | (A.X <= 8)))
    s.add("VEC", A.enum("scalar", "vec2", "vec4"), A.X <= A.P(1))
    _check_against_oracle(Space, s)
    with Space(s) as sp:
        sp.generate()
        rows = sp.decode(torch.arange(sp.size(), dtype=torch.int64, device="cuda"))
        named = sp.to_named(rows)
        assert named[0] == {"MEM": "global", "TS": 1, "VEC": "scalar"}
        assert {r["MEM"] for r in named} == {"global", "local", "private"}
        assert all(r["TS"] <= 8 or r["MEM"] == "local" for r in named)


def _seg_bound_spec(kind, order, top=1500):
    """Wide divisibility chains whose candidate sets put 0, negatives and large values in
    different warp-tile segments (sorted, reversed, shuffled): the per-segment |x| bounds of
    the hot filter (x | n needs |x| <= |n|, d | x needs |x| >= |d|, 0 passes both) must not
    drop an accepted pair."""
    import random
    vals = list(range(-40, 0)) + [0] + list(range(1, top))
    if order == "reversed":
        vals = vals[::-1]
    elif order == "shuffled":
        random.Random(7).shuffle(vals)
    s = A.Spec(f"segbound_{kind}_{order}_{top}")
    alias = A.divides if kind == "divx" else A.is_multiple_of
    s.add("a", A.interval(-3, 40))
    s.add("b", A.set_(*vals), alias(s.P("a")))
    s.add("c", A.set_(*vals), alias(s.P("b")))
    return s


@pytest.mark.parametrize("kind", ["divx", "mulx"])
@pytest.mark.parametrize("order", ["sorted", "reversed", "shuffled"])
def test_segment_bounds_parity(Space, kind, order):
    _check_against_oracle(Space, _seg_bound_spec(kind, order), decode_all_max=200_000)


@pytest.mark.parametrize("kind", ["divx", "mulx"])
@pytest.mark.parametrize("order", ["sorted", "shuffled"])
def test_segment_bounds_parity_eight_segments(Space, kind, order):
    """r = 7341 candidates: both the divisor (x | n) and the multiples (d | x) hot filters run
    8 segments of 1024 (the 8th, partial, segment included); leaves compared element-wise."""
    from paper_conf_hpdc_raschg18_b200 import _lib as L
    spec = _seg_bound_spec(kind, order, top=7301)
    with Space(spec) as sp:
        sp.generate()
        assert [x["nseg"] for x in sp.stats()] == [0, 8, 8]
    _check_against_oracle(Space, spec, decode_all_max=200_000)
    _check_against_oracle(Space, spec, decode_all_max=200_000, extra_flags=L.ATF_FLAG_NO_SEG_BOUNDS)


def test_segment_bounds_skip_work_not_results(Space):
    """ATF_FLAG_TIMING statistics: evaluated pairs never exceed the spec's f_{k-1} r_k, equal it
    on levels without the filter, and fall below it where nodes' values exclude whole segments
    (C5's divisor chain: deep levels hold small values).  Level sizes stay the oracle's
    (C5 closed form, Piltz divisor sums)."""
    from paper_conf_hpdc_raschg18_b200 import _lib as L
    spec = A.c5_chains(4096, 4)
    with Space(spec, flags=L.ATF_FLAG_TIMING | L.ATF_FLAG_SERIAL_GROUPS) as sp:
        sp.generate()
        st = sp.stats()
        assert all(0 < x["pairs"] <= x["evals"] for x in st if x["evals"])
        g0 = [x for x in st if x["group"] == 0]
        assert g0[-1]["pairs"] < g0[-1]["evals"] // 2
        assert sp.level_sizes(0) == cf.piltz_D(4096, 4)


# ---------------------------------------------------------------- u128 indices (S >= 2^64)
def _big_spec():
    """Six independent groups (x_i in [1,3000], y_i | x_i): S = (sum_{n<=3000} tau(n))^6 ~ 2^88."""
    s = A.Spec("six_divisor_groups")
    for i in range(6):
        s.add(f"x{i}", A.interval(1, 3000))
        s.add(f"y{i}", A.interval(1, 3000), A.divides(s.P(f"x{i}")))
    return s


def test_decode_u128_indices_against_oracle_leaves(Space):
    """decode_range / decode_indices128 (P:229-231 index access, P:280 spaces beyond 2^64):
    index -> mixed-radix digits (group 0 most significant, reading #11) computed here in Python
    integers -> the oracle's leaf rows of every group, element by element."""
    spec = _big_spec()
    ref = orc.info(spec, threads=8)
    sizes = [g["size"] for g in ref["groups"]]
    S = int(ref["S"])
    assert S >= 1 << 64
    leaves = [orc.leaves(spec, g, 2) for g in range(6)]

    def want(indices):
        rows = []
        for i in indices:
            dig, rem = [], i
            for z in reversed(sizes):
                dig.append(rem % z)
                rem //= z
            dig.reverse()
            rows.append([int(v) for g in range(6) for v in leaves[g][dig[g]]])
        return np.array(rows, dtype=np.int32).T
    gen = np.random.default_rng(5)
    with Space(spec) as sp:
        sp.generate()
        assert sp.size() == S
        for first in (0, S // 3, (1 << 64) - 7, S - 50):
            got = sp.decode_range(first, 50).cpu().numpy()
            assert np.array_equal(got, want(range(first, first + 50))), first
        idx = [int(gen.integers(0, 1 << 62)) * (1 << 26) % S for _ in range(2000)] + [S - 1, 0]
        lo = torch.tensor([((i & ((1 << 64) - 1)) ^ (1 << 63)) - (1 << 63) for i in idx], dtype=torch.int64).cuda()
        hi = torch.tensor([i >> 64 for i in idx], dtype=torch.int64).cuda()
        assert np.array_equal(sp.decode128(lo, hi).cpu().numpy(), want(idx))
        from paper_conf_hpdc_raschg18_b200 import AtfError
        with pytest.raises(AtfError):
            sp.decode_range(S - 2, 4)


def test_exhaustive_search_beyond_2_64(Space):
    """ExhaustiveSearch walks any space in index order through decode_range."""
    from paper_conf_hpdc_raschg18_b200 import explore
    spec = _big_spec()
    with Space(spec) as sp:
        sp.generate()
        t = explore.ExhaustiveSearch()
        t.initialize(sp)
        t.next = sp.size() - 10
        a = t.get_next_configs(4)
        b = t.get_next_configs(100)
        assert a.shape[1] == 4 and b.shape[1] == 6
        assert torch.equal(torch.cat([a, b], 1), sp.decode_range(sp.size() - 10, 10))


# ---------------------------------------------------------------- allocation failure (fault injection)
def test_allocator_failure_is_reported_and_space_destroys_cleanly(Space):
    """SURVEY.md §5 failure detection: the device allocator hook returns NULL at the k-th request
    (k = 0, 1, ... up to every allocation a generation makes).  generate must return ATF_ERR_OOM
    (never crash or hang), destroy must free every block that was handed out, and a later
    generation of the same spec with a working allocator is still exact."""
    import ctypes as C
    from paper_conf_hpdc_raschg18_b200 import _lib as LL
    from paper_conf_hpdc_raschg18_b200.space import _range_struct
    spec = A.c3_xgemm((12, 30, 8))
    ref = int(orc.info(spec)["S"])
    stream = torch.cuda.current_stream()

    def run(fail_at):
        live, count = {}, [0]

        def _alloc(nbytes, _st, _ctx):
            count[0] += 1
            if count[0] - 1 == fail_at:
                return None
            t = torch.empty(int(nbytes), dtype=torch.uint8, device="cuda")
            live[t.data_ptr()] = t
            return t.data_ptr()

        def _free(ptr, _n, _st, _ctx):
            assert ptr in live, "free of a block the hook never handed out"
            live.pop(ptr)

        acb, fcb = LL.ALLOC_FN(_alloc), LL.FREE_FN(_free)
        opts = LL.atf_space_opts(0, stream.cuda_stream, acb, fcb, None, 0)
        h = C.c_void_p()
        LL.check(LL.atf_space_create(C.byref(opts), C.byref(h)))
        keep = []
        for p in spec.params:
            rs, k = _range_struct(p.range)
            keep.append(k)
            pid = C.c_int32()
            LL.check(LL.atf_space_add_param(h, p.name.encode(), C.byref(rs), C.byref(pid)), h)
            for code in p.constraints:
                arr = (C.c_int32 * len(code))(*code)
                LL.check(LL.atf_space_add_constraint(h, pid.value, arr, len(code)), h)
        st = LL.atf_space_generate(h)
        S = None
        if st == 0:
            lo, hi = C.c_uint64(), C.c_uint64()
            LL.check(LL.atf_space_size(h, C.byref(lo), C.byref(hi)), h)
            S = lo.value
        LL.atf_space_destroy(h)
        torch.cuda.synchronize()
        assert not live, f"{len(live)} blocks leaked (fail_at={fail_at})"
        return st, S, count[0]

    st, S, total = run(-1)
    assert st == 0 and S == ref and total >= 3
    for k in range(total):
        st, S, _ = run(k)
        assert st == -2, (k, st)          # ATF_ERR_OOM
    assert run(-1)[:2] == (0, ref)


# ---------------------------------------------------------------- balanced multi-GPU generation
def _dist_check(Space, spec, world, flags=0, gens=1, streams=False):
    """generate_dist on `world` virtual ranks (spaces of this process): global sizes = the oracle's,
    every level's rank slices (records, by offset) concatenate to the single-GPU level, and the
    ranks' CSR slices (by csr_offset) concatenate to the single-GPU CSR; every rank expanded
    ~1/world of every level's parents (the balance rule).  `gens` generations of the same spaces
    (the third and later replay: one all-gather each, device flags between the ranks' streams;
    `streams`: one CUDA stream per rank, concurrent ranks).  Returns the all-gather calls per
    generation."""
    from paper_conf_hpdc_raschg18_b200.shard import virtual_ranks
    ref = orc.info(spec, threads=8)
    with Space(spec, flags=flags) as one:
        one.generate()
        G = one.num_groups()
        want = {(g, k): tuple(t.clone() if t is not None else None for t in one.level_tensors(g, k))
                for g in range(G) for k in range(one.num_levels(g))}
        sizes = one.group_sizes()
    spaces = [Space(spec, flags=flags, stream=torch.cuda.Stream() if streams else None) for _ in range(world)]
    calls = []
    try:
        for i in range(gens):
            vag = virtual_ranks(spaces)
            calls.append(vag.calls[0])
            _dist_compare(spaces, want, sizes, ref, world, check_balance=i == 0)
    finally:
        for sp in spaces:
            sp.close()
    return calls


def _dist_compare(spaces, want, sizes, ref, world, check_balance=True):
    """Every rank's slices against the single-GPU arrays.  A replicated level is held whole by the
    ranks of its group (all ranks in the first generation; after one, groups may own subsets of
    the ranks); a distributed level's non-empty slices are contiguous by offset and
    concatenate to it; the CSR slices likewise.  `check_balance`: every rank's parent slice is
    floor / ceil of f_k / world (the first generation's rule)."""
    assert sizes == [g["size"] for g in ref["groups"]]
    for sp in spaces:
        assert sp.group_sizes() == sizes
        assert sp.size() == int(ref["S"])
    for (g, k), (wrec, wcsr) in want.items():
        parts, cparts = [], []
        for sp in spaces:
            v = sp.level_view(g, k)
            rec, csr = sp.level_tensors(g, k)
            if rec is not None and rec.shape[0]:
                parts.append((v["offset"], rec))
            if csr is not None:
                cparts.append((v["csr_offset"], csr, v["offset"], 0 if rec is None else rec.shape[0]))
        n = wrec.shape[0] if wrec is not None else 0
        if not parts:
            assert n == 0, (g, k)
        elif world > 1 and len(parts) > 1 and all(off == 0 and r.shape[0] == n for off, r in parts):
            for _, r in parts:  # replicated: every holder has all of it
                assert torch.equal(r, wrec), (g, k)
        else:
            parts.sort(key=lambda t: t[0])
            pos = 0
            for off, rec in parts:
                assert off == pos, (g, k)
                pos += rec.shape[0]
            assert torch.equal(torch.cat([r for _, r in parts]), wrec), (g, k)
        if wcsr is None:
            continue
        full = [c for c in cparts if c[0] == 0 and c[1].shape[0] == n + 1]
        sl = [c for c in cparts if c[1].shape[0] > 1]
        if world > 1 and len(full) > 1 and len(full) == len(sl):
            for c in full:
                assert torch.equal(c[1], wcsr), ("csr", g, k)
            continue
        if not sl:
            assert n == 0, ("csr", g, k)
            continue
        sl.sort(key=lambda t: t[0])
        pos = 0
        for c in sl:
            assert c[0] == pos, ("csr offset", g, k)
            pos += c[1].shape[0] - 1
        got = torch.cat([c[1][:-1] for c in sl] + [sl[-1][1][-1:]])
        assert torch.equal(got, wcsr), ("csr", g, k)
        if check_balance:
            # a rank's parent slice (CSR not covering exactly its own nodes, i.e. not inside a fused
            # tail) is floor/ceil of f_k / world
            for c in cparts:
                if (c[0], c[1].shape[0] - 1) != (c[2], c[3]):
                    assert abs((c[1].shape[0] - 1) - n / world) <= 1, (g, k)


@pytest.mark.parametrize("world", [2, 3, 8])
@pytest.mark.parametrize("name", ["C5-300x4", "C3-IS1", "C2-256", "C5-4096x3", "fig1", "C1"])
def test_dist_virtual_ranks_match_single_gpu(Space, world, name):
    _dist_check(Space, SMALL[name](), world)


@pytest.mark.parametrize("seed", range(0, 40, 4))
def test_dist_virtual_ranks_fuzz(Space, seed):
    _dist_check(Space, A.random_spec(seed), 3)
    _dist_check(Space, A.random_wide_spec(seed), 2)


def test_dist_virtual_ranks_headline_flags(Space):
    from paper_conf_hpdc_raschg18_b200 import _lib as L
    _dist_check(Space, A.c5_chains(4096, 4), 4, flags=L.ATF_FLAG_NO_SEG_BOUNDS)
    _dist_check(Space, A.c3_xgemm((20, 96, 8)), 4, flags=L.ATF_FLAG_NO_JIT)


@pytest.mark.parametrize("world", [1, 2, 3])
@pytest.mark.parametrize("name", ["C5-300x4", "C3-IS1", "C2-256", "C5-4096x3", "fig1"])
def test_dist_replay_virtual_ranks(Space, world, name):
    """Steady state of generate_dist: the first generation synchronises per round, the second
    sizes every level from the log, the third and later replay with device flags (one all-gather
    per generation, the verdicts) -- every generation identical to the single-GPU space."""
    from paper_conf_hpdc_raschg18_b200 import _lib as L
    # default (rank subsets from generation 2): the assignment changes once, so the replay starts a
    # generation later (fresh log, log-sized, then replays)
    calls = _dist_check(Space, SMALL[name](), world, gens=5, streams=True)
    assert calls[3] == calls[4] == 1, calls
    # the plain partition (every group on every rank): generation 2 repeats generation 1's rounds
    calls = _dist_check(Space, SMALL[name](), world, flags=L.ATF_FLAG_DIST_NO_SUBSETS, gens=4, streams=True)
    assert calls[2] == calls[3] == 1, calls
    assert calls[0] == calls[1], calls   # (0 when every level is replicated)


@pytest.mark.parametrize("seed", range(0, 24, 5))
def test_dist_replay_fuzz(Space, seed):
    calls = _dist_check(Space, A.random_spec(seed), 3, gens=4, streams=True)
    assert calls[3] == 1, calls


def test_dist_replay_headline_flags(Space):
    from paper_conf_hpdc_raschg18_b200 import _lib as L
    calls = _dist_check(Space, A.c5_chains(4096, 4), 4, flags=L.ATF_FLAG_NO_SEG_BOUNDS, gens=4, streams=True)
    assert calls[3] == 1, calls
    plain = L.ATF_FLAG_DIST_NO_SUBSETS
    calls = _dist_check(Space, A.c5_chains(4096, 5), 2, flags=L.ATF_FLAG_NO_SEG_BOUNDS | plain, gens=3, streams=True)
    assert calls == [2, 2, 1], calls   # levels 4, 5 distributed; then the replay
    calls = _dist_check(Space, A.c5_chains(4096, 5), 2, flags=L.ATF_FLAG_NO_REPLAY | plain, gens=3, streams=True)
    assert calls == [2, 2, 2], calls   # replay off: one all-gather per distributed round every time


@pytest.mark.parametrize("world", [2, 3, 8])
@pytest.mark.parametrize("name", ["C5-300x4", "C5-4096x3", "C3-IS1", "fig1"])
def test_dist_group_subsets(Space, world, name):
    """Rank subsets (the default; ATF_FLAG_DIST_SUBSETS is a no-op since round 2): from the second
    generation each group owns a subset of the ranks
    (in proportion to its candidate pairs); the non-members follow its rounds with empty slices.
    Every generation identical to the single-GPU space; the fourth and later replay."""
    from paper_conf_hpdc_raschg18_b200 import _lib as L
    calls = _dist_check(Space, SMALL[name](), world, flags=L.ATF_FLAG_DIST_SUBSETS, gens=5, streams=True)
    assert calls[-1] == calls[-2] == 1, calls


def test_dist_two_processes_cuda_ipc(Space, tmp_path):
    """Two processes on the one GPU, gloo all-gather: the parent slices cross processes through
    CUDA IPC (cudaIpcGetMemHandle / OpenMemHandle), the path every rank of an 8-GPU node uses."""
    import subprocess
    import sys
    script = tmp_path / "ipc_ranks.py"
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    script.write_text(f"""
import os, sys, torch, numpy as np
sys.path.insert(0, {root!r})
import torch.distributed as dist
import atfspec as A
from paper_conf_hpdc_raschg18_b200 import Space
from paper_conf_hpdc_raschg18_b200.shard import generate_balanced
dist.init_process_group("gloo")
r = dist.get_rank()
torch.cuda.set_device(0)
calls = []
def ag(b):
    calls.append(len(b))
    t = torch.frombuffer(bytearray(b), dtype=torch.uint8)
    o = torch.empty(2 * t.numel(), dtype=torch.uint8)
    dist.all_gather_into_tensor(o, t)
    return o.numpy().tobytes()
with Space(A.c5_chains(300, 4), stream=torch.cuda.Stream()) as sp:
    ncalls = []
    for _ in range(5):   # synchronous; rank subsets: fresh log, log-sized, then two replays (device flags across processes)
        n0 = len(calls)
        sp.generate_dist(r, 2, ag)
        ncalls.append(len(calls) - n0)
    torch.cuda.synchronize()
    out = {{"sizes": sp.group_sizes(), "calls": ncalls}}
    for g in range(sp.num_groups()):
        for k in range(sp.num_levels(g)):
            v = sp.level_view(g, k)
            rec, csr = sp.level_tensors(g, k)
            out[f"r{{g}}_{{k}}"] = (v["offset"], rec.cpu().numpy() if rec is not None else np.zeros((0, 1), np.uint32))
            if csr is not None:
                out[f"c{{g}}_{{k}}"] = (v["csr_offset"], csr.cpu().numpy())
    np.save({str(tmp_path)!r} + f"/rank{{r}}.npy", out, allow_pickle=True)
dist.destroy_process_group()
""")
    env = dict(os.environ, MASTER_ADDR="127.0.0.1")
    p = subprocess.run([sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node=2",
                        "--master-addr", "127.0.0.1", "--master-port", "29531", str(script)],
                       capture_output=True, text=True, timeout=600, env=env)
    assert p.returncode == 0, p.stdout[-3000:] + p.stderr[-3000:]
    res = [np.load(tmp_path / f"rank{r}.npy", allow_pickle=True).item() for r in range(2)]
    spec = A.c5_chains(300, 4)
    for r in range(2):
        assert res[r]["calls"][3] == res[r]["calls"][4] == 1, res[r]["calls"]
    with Space(spec) as one:
        one.generate()
        assert res[0]["sizes"] == res[1]["sizes"] == one.group_sizes()
        for g in range(one.num_groups()):
            for k in range(one.num_levels(g)):
                rec, csr = one.level_tensors(g, k)
                rec = rec.cpu().numpy()
                parts = sorted([res[r][f"r{g}_{k}"] for r in range(2) if res[r][f"r{g}_{k}"][1].shape[0]],
                               key=lambda t: t[0])
                if len(parts) == 2 and all(off == 0 and p.shape[0] == rec.shape[0] for off, p in parts):
                    assert all(np.array_equal(p, rec) for _, p in parts)   # replicated on both ranks
                elif parts:
                    assert np.array_equal(np.concatenate([p for _, p in parts]), rec)
                else:
                    assert rec.shape[0] == 0
                if csr is not None:
                    csr = csr.cpu().numpy()
                    cp = sorted([res[r][f"c{g}_{k}"] for r in range(2) if f"c{g}_{k}" in res[r] and
                                 res[r][f"c{g}_{k}"][1].shape[0] > 1], key=lambda t: t[0])
                    if len(cp) == 2 and all(off == 0 and c.shape[0] == csr.shape[0] for off, c in cp):
                        assert all(np.array_equal(c, csr) for _, c in cp)
                    elif cp:
                        assert np.array_equal(np.concatenate([c[1][:-1] for c in cp] + [cp[-1][1][-1:]]), csr)


def test_float_parameters_by_position(Space):
    """Float-valued parameters (NEXT-3, "float") by position index: a tolerance in
    float_interval(0.25, 2.0, 0.25) constrained through its (monotone) positions together with
    integer parameters; the space equals the oracle's (which sees the same positions), and
    to_named gives the float values."""
    s = A.Spec("float_space")
    tol = A.float_interval(0.25, 2.0, 0.25)
    s.add("TS", A.interval(1, 64), A.divides(64))
    s.add("TOL", tol, (A.X <= A.float_code(tol, 1.0)) | (s.P("TS") >= 16))
    s.add("UNROLL", A.interval(1, 8), A.divides(s.P("TS")) & (A.X * (s.P("TOL") + 1) <= 16))
    _check_against_oracle(Space, s)
    with Space(s) as sp:
        sp.generate()
        named = sp.to_named(sp.decode(torch.arange(sp.size(), dtype=torch.int64, device="cuda")))
        assert all(isinstance(r["TOL"], float) for r in named)
        assert all(r["TOL"] <= 1.0 or r["TS"] >= 16 for r in named)
        assert {r["TOL"] for r in named} == {0.25 * i for i in range(1, 9)}


@pytest.mark.parametrize("name", ["C2-256", "C3-IS1", "C5-300x4", "C3-12x30x8"])
def test_sync_rounds_and_dfs_tail_count_parity(Space, name):
    """The A/B alternatives stay exact: one synchronising level round for all groups
    (atf_test_set_async_rounds(0)) instead of per-group rounds, and the depth-first tail count
    (atf_test_set_tail_product(0)) instead of the product count."""
    from paper_conf_hpdc_raschg18_b200 import _lib as L
    L.check(L.atf_test_set_async_rounds(0))
    L.check(L.atf_test_set_tail_product(0))
    L.check(L.atf_test_set_tail_leaf_direct(1))   # leaves straight to global memory in every tail
    try:
        _check_against_oracle(Space, SMALL[name]())
        L.check(L.atf_test_set_tail_leaf_direct(0))   # leaves staged in every tail
        _check_against_oracle(Space, SMALL[name]())
    finally:
        L.check(L.atf_test_set_async_rounds(1))
        L.check(L.atf_test_set_tail_product(1))
        L.check(L.atf_test_set_tail_leaf_direct(2))
