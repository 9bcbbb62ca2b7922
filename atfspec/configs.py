"""The parameter specifications of BASELINE.json's configs and the paper's examples.

Every spec here is deterministic: the "value distribution" of this workload is
the constraint structure itself.  Citations: P:n = PAPER.md
line n.  Readings of unstated details are the SURVEY.md §8(c) readings, listed
in DESIGN.md.
"""
from __future__ import annotations

from . import (Spec, X, C, DIVIDES, MULOF, divides, is_multiple_of, interval, set_, pow2)

__all__ = ["c1_toy", "c2_xgemm_direct", "c3_xgemm", "c5_chains", "saxpy", "fig1",
           "IS_SHAPES", "CONFIGS", "config_spec", "c4_indices_seed"]

# Caffe GEMM shapes IS1-IS4: (M, K) x (K, N) -> (M, N, K)
IS_SHAPES = {
    "IS1": (20, 576, 1),    # 20x1  . 1x576
    "IS2": (20, 576, 25),   # 20x25 . 25x576
    "IS3": (50, 64, 1),     # 50x1  . 1x64
    "IS4": (10, 500, 64),   # 10x64 . 64x500
}


def c1_toy() -> Spec:
    """configs[0]: TS_M, TS_N in 1..64, TS_M|64, TS_N|64, TS_M*TS_N <= 1024."""
    s = Spec("C1_toy_2d_tiling")
    m = s.add("TS_M", interval(1, 64), divides(64))
    s.add("TS_N", interval(1, 64), divides(64) & ((s.P("TS_M") * X) <= 1024))
    return s


def c2_xgemm_direct(n: int = 256, implied: bool = True, anchored: bool = True) -> Spec:
    """configs[1]: CLBlast XgemmDirect space, M=N=K=n (reading #12 in DESIGN.md).

    c1 KWID|WGD; c2 MDIMCD*VWMD|WGD; c3 NDIMCD*VWND|WGD; c4 MDIMAD*VWMD|WGD;
    c5 NDIMBD*VWND|WGD; c6 (MDIMCD*NDIMCD/MDIMAD)|WGD; c7 (MDIMCD*NDIMCD/NDIMBD)|WGD;
    anchors WGD|M, WGD|N; implied early-prune {MDIMCD,NDIMCD,MDIMAD,NDIMBD}|WGD.
    """
    s = Spec(f"C2_xgemm_direct_{n}" + ("" if implied else "_noimplied") + ("" if anchored else "_unanchored"))
    M = N = n
    s.add("WGD", interval(1, n), *( [divides(M) & divides(N)] if anchored else []))
    WGD = s.P("WGD")
    s.add("MDIMCD", interval(1, n), divides(WGD) if implied else None)
    s.add("NDIMCD", interval(1, n), divides(WGD) if implied else None)
    MDIMCD, NDIMCD = s.P("MDIMCD"), s.P("NDIMCD")
    c6 = MULOF(WGD, (MDIMCD * NDIMCD) // X)
    s.add("MDIMAD", interval(1, n), (divides(WGD) & c6) if implied else c6)
    s.add("NDIMBD", interval(1, n), (divides(WGD) & c6) if implied else c6)
    s.add("KWID", interval(1, n), divides(WGD))
    MDIMAD, NDIMBD = s.P("MDIMAD"), s.P("NDIMBD")
    s.add("VWMD", set_(1, 2, 4, 8), DIVIDES(MDIMCD * X, WGD) & DIVIDES(MDIMAD * X, WGD))
    s.add("VWND", set_(1, 2, 4, 8), DIVIDES(NDIMCD * X, WGD) & DIVIDES(NDIMBD * X, WGD))
    s.add("PADA", set_(0, 1))
    s.add("PADB", set_(0, 1))
    return s


def c3_xgemm(shape="IS2", anchored: bool = False) -> Spec:
    """configs[2]: CLBlast Xgemm 14-parameter space, ranges 1..input size (reading #13).

    Per-dimension ranges: MWG, MDIMC, MDIMA in 1..M; NWG, NDIMC, NDIMB in 1..N;
    KWG, KWI in 1..K.  No MWG|M anchors.  ``anchored=True`` is the
    cross-check variant: MWG|M, NWG|N, KWG|K and all ranges 1..max(M,N,K).
    """
    if isinstance(shape, str):
        M, N, K = IS_SHAPES[shape]
        tag = shape
    else:
        M, N, K = shape
        tag = f"{M}x{N}x{K}"
    s = Spec(f"C3_xgemm_{tag}" + ("_anchored" if anchored else ""))
    R = max(M, N, K)
    rm, rn, rk = (R, R, R) if anchored else (M, N, K)
    s.add("MWG", interval(1, rm), divides(M) if anchored else None)
    s.add("NWG", interval(1, rn), divides(N) if anchored else None)
    s.add("KWG", interval(1, rk), divides(K) if anchored else None)
    MWG, NWG, KWG = s.P("MWG"), s.P("NWG"), s.P("KWG")
    s.add("MDIMC", interval(1, rm), divides(MWG))
    s.add("NDIMC", interval(1, rn), divides(NWG))
    MDIMC, NDIMC = s.P("MDIMC"), s.P("NDIMC")
    s.add("MDIMA", interval(1, rm), divides(MWG) & MULOF(KWG, (MDIMC * NDIMC) // X))
    s.add("NDIMB", interval(1, rn), divides(NWG) & MULOF(KWG, (MDIMC * NDIMC) // X))
    s.add("KWI", interval(1, rk), divides(KWG))
    MDIMA, NDIMB = s.P("MDIMA"), s.P("NDIMB")
    s.add("VWM", set_(1, 2, 4, 8), DIVIDES(MDIMC * X, MWG) & DIVIDES(MDIMA * X, MWG))
    s.add("VWN", set_(1, 2, 4, 8), DIVIDES(NDIMC * X, NWG) & DIVIDES(NDIMB * X, NWG))
    for b in ("STRM", "STRN", "SA", "SB"):
        s.add(b, set_(0, 1))
    return s


def c5_chains(R: int = 4096, length: int = 8) -> Spec:
    """configs[4]: 24 parameters in 3 independent chains (synthetic, north star).

    G0 x0..x7 in [1,R], x_k divides x_{k-1};  G1 y0..y7 in [1,R], y_k is a
    multiple of y_{k-1};  G2 z0..z7 in interval(2,R,2), z_k divides z_{k-1}.
    """
    s = Spec(f"C5_chains_{R}x{length}")
    for pfx, rng, alias in (("x", interval(1, R), divides),
                            ("y", interval(1, R), is_multiple_of),
                            ("z", interval(2, R, 2), divides)):
        prev = None
        for k in range(length):
            cur = s.add(f"{pfx}{k}", rng, alias(s.P(f"{pfx}{k-1}")) if prev is not None else None)
            prev = cur
    return s


def saxpy(n: int) -> Spec:
    """The paper's running example: WPT in [1,N], WPT|N; LS in [1,N], LS|(N/WPT)."""
    s = Spec(f"saxpy_{n}")
    s.add("WPT", interval(1, n), divides(n))
    s.add("LS", interval(1, n), divides(C(n) // s.P("WPT")))
    return s


def fig1() -> Spec:
    """Fig. 1: tp1..tp4 in {1,2}; tp2: divides(tp1); tp4: divides(tp3)."""
    s = Spec("fig1")
    s.add("tp1", set_(1, 2))
    s.add("tp2", set_(1, 2), divides(s.P("tp1")))
    s.add("tp3", set_(1, 2))
    s.add("tp4", set_(1, 2), divides(s.P("tp3")))
    return s


def c4_indices_seed() -> int:
    """configs[3]: idx_i = splitmix64(0x41544617 + i) mod S."""
    return 0x41544617


CONFIGS = {
    "C1": c1_toy,
    "C2": lambda: c2_xgemm_direct(256),
    "C3-IS1": lambda: c3_xgemm("IS1"),
    "C3-IS2": lambda: c3_xgemm("IS2"),
    "C3-IS3": lambda: c3_xgemm("IS3"),
    "C3-IS4": lambda: c3_xgemm("IS4"),
    "C5": c5_chains,
}


def config_spec(name: str) -> Spec:
    return CONFIGS[name]()
