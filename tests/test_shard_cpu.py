"""Host logic of the multi-GPU shard layer on CPU.

* shard_slice: the rank slices of a cut level partition it contiguously and are balanced
  by child counts;
* world_size-2 gloo run of the shard protocol: each rank takes its slice of the cut
  level of the C5 chain space (small R), counts its nodes per level, the counts are
  all-gathered through paper_conf_hpdc_raschg18_b200.shard.all_gather_counts (the same
  call bench.py makes over NCCL), and shard_offsets turns them into global offsets and
  totals, which must equal the oracle's per-level sizes (P:235-247 groups; Piltz counts).
"""
import ctypes as C
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import atfspec as A


def _lib():
    from paper_conf_hpdc_raschg18_b200 import _lib as L
    return L


def _slice(csr, rank, world):
    L = _lib()
    arr = (C.c_uint64 * len(csr))(*[int(v) for v in csr])
    lo, hi = C.c_uint64(), C.c_uint64()
    L.check(L.atf_test_shard_slice(arr, len(csr) - 1, rank, world, C.byref(lo), C.byref(hi)))
    return lo.value, hi.value


def _offsets(allc, rank):
    L = _lib()
    world, n = len(allc), len(allc[0])
    flat = (C.c_int64 * (world * n))(*[int(c) for row in allc for c in row])
    before, tot = (C.c_uint64 * n)(), (C.c_uint64 * n)()
    L.check(L.atf_test_shard_offsets(flat, world, n, rank, before, tot))
    return list(before), list(tot)


@pytest.mark.parametrize("seed", range(6))
@pytest.mark.parametrize("world", [1, 2, 3, 4, 8])
def test_slices_partition_and_balance(seed, world):
    rng = np.random.default_rng(seed * 131 + world)
    n = int(rng.integers(0, 300))
    kind = seed % 3
    if kind == 0:
        cnt = rng.integers(0, 20, n)
    elif kind == 1:
        cnt = np.zeros(n, dtype=np.int64)
        if n:
            cnt[rng.integers(0, n)] = 1000  # one huge subtree
    else:
        cnt = rng.geometric(0.05, n) * (rng.random(n) < 0.3)
    csr = np.concatenate([[0], np.cumsum(cnt)]).astype(np.uint64)
    T = int(csr[-1])
    prev_hi = 0
    mx = int(cnt.max()) if n else 0
    for r in range(world):
        lo, hi = _slice(csr, r, world)
        assert lo == prev_hi and lo <= hi <= n
        prev_hi = hi
        share = int(csr[hi] - csr[lo])
        assert abs(share - T / world) <= mx + 1, (r, share, T / world, mx)
    assert prev_hi == n


def test_offsets_exclusive_scan():
    allc = [[3, 0, 7], [1, 5, 0], [0, 2, 9]]
    for r in range(3):
        before, tot = _offsets(allc, r)
        assert tot == [4, 7, 16]
        assert before == [sum(allc[q][i] for q in range(r)) for i in range(3)]


# ---------------------------------------------------------------- gloo, world 2
R, LEN, CUT = 60, 4, 1


def _chain_tree(spec):
    """Per group: list of levels, each a list of path tuples (range positions), built by
    plain nested loops from the spec's own ranges (chain: x_k | x_{k-1} for G0/G2,
    x_k multiple of x_{k-1} for G1 — configs.c5_chains)."""
    groups = []
    for g in range(3):
        params = spec.params[g * LEN:(g + 1) * LEN]
        vals = [list(range(p.range["begin"], p.range["end"] + 1, p.range.get("step", 1))) for p in params]
        levels = [[(j,) for j in range(len(vals[0]))]]
        for k in range(1, LEN):
            nxt = []
            for path in levels[-1]:
                pv = vals[k - 1][path[-1]]
                for j, x in enumerate(vals[k]):
                    ok = (pv % x == 0) if g != 1 else (x % pv == 0)
                    if ok:
                        nxt.append(path + (j,))
            levels.append(nxt)
        groups.append(levels)
    return groups


def _children_csr(levels, k):
    parents = levels[k]
    idx = {p: i for i, p in enumerate(parents)}
    cnt = np.zeros(len(parents), dtype=np.int64)
    for c in levels[k + 1]:
        cnt[idx[c[:-1]]] += 1
    return np.concatenate([[0], np.cumsum(cnt)]).astype(np.uint64)


def _rank_main(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_hpdc_raschg18_b200.shard import all_gather_counts
        spec = A.c5_chains(R, LEN)
        tree = _chain_tree(spec)
        counts, first = [], []
        for levels in tree:
            csr = _children_csr(levels, CUT)
            lo, hi = _slice(csr, rank, world)
            mine = set(levels[CUT][lo:hi])
            for k, lev in enumerate(levels):
                if k <= CUT:  # replicated prefix: counted once (rank 0)
                    counts.append(len(lev) if rank == 0 else 0)
                    first.append(0)
                else:
                    pos = [i for i, p in enumerate(lev) if p[:CUT + 1] in mine]
                    counts.append(len(pos))
                    first.append(pos[0] if pos else None)
                    # the rank's nodes are one contiguous run of the canonical order
                    assert pos == list(range(pos[0], pos[0] + len(pos))) if pos else True
        allc = all_gather_counts(counts)
        before, tot = _offsets(allc, rank)
        q.put((rank, counts, first, allc, before, tot))
    finally:
        dist.destroy_process_group()


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def test_gloo_world2_shard_protocol(oracle_bin):
    from oracle import run as orc
    spec = A.c5_chains(R, LEN)
    ref = orc.info(spec)
    want = [lv["f"] for grp in ref["groups"] for lv in grp["levels"]]
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_rank_main, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = {}
    for _ in range(world):
        rank, counts, first, allc, before, tot = q.get(timeout=240)
        res[rank] = (counts, first, allc, before, tot)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    for rank, (counts, first, allc, before, tot) in res.items():
        assert allc == [res[r][0] for r in range(world)]       # the all-gather is rank-major
        assert tot == want, (tot, want)                         # global level sizes = oracle f_k
        for i, f in enumerate(first):
            if f is not None and counts[i]:
                assert before[i] == f                            # global offset of this rank's run


# ---------------------------------------------------------------- balanced per-level protocol, gloo world 2
def _balanced_rank_main(rank, world, port, q):
    """atf_space_generate_dist's protocol restated on the CPU (plain loops over the chain tree):
    level k is expanded from the parent slice [r F / N, (r+1) F / N) of level k - 1, the ranks
    all-gather one byte record per level through shard._allgather_bytes (gloo), and the next
    parent slice is taken from the concatenation of the ranks' children."""
    import struct
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_hpdc_raschg18_b200.shard import _allgather_bytes
        spec = A.c5_chains(R, LEN)
        out = []
        for g in range(3):
            params = spec.params[g * LEN:(g + 1) * LEN]
            vals = [list(range(p.range["begin"], p.range["end"] + 1, p.range.get("step", 1))) for p in params]
            frontier = [()]
            F = 1
            per_level = []
            for k in range(LEN):
                lo, hi = F * rank // world, F * (rank + 1) // world
                kids = []
                for path in frontier[lo:hi]:
                    for j, x in enumerate(vals[k]):
                        if k == 0:
                            ok = True
                        else:
                            pv = vals[k - 1][path[-1]]
                            ok = (pv % x == 0) if g != 1 else (x % pv == 0)
                        if ok:
                            kids.append(path + (j,))
                rec = struct.pack("<q", len(kids))
                allb = _allgather_bytes(rec)
                counts = [struct.unpack_from("<q", allb, 8 * r)[0] for r in range(world)]
                # the real library copies the parent slice from the ranks' arenas; here every rank
                # rebuilds the level from the gathered children (small spec)
                gathered = _allgather_bytes(repr(kids).encode().ljust(1 << 20))
                full = []
                for r in range(world):
                    full += eval(gathered[r << 20:(r + 1) << 20].rstrip())
                assert len(full) == sum(counts)
                per_level.append((hi - lo, sum(counts), sum(counts[:rank]), kids[:1]))
                frontier, F = full, len(full)
            out.append(per_level)
        q.put((rank, out))
    finally:
        dist.destroy_process_group()


def test_gloo_world2_balanced_protocol(oracle_bin):
    from oracle import run as orc
    spec = A.c5_chains(R, LEN)
    ref = orc.info(spec)
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_balanced_rank_main, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = {}
    for _ in range(world):
        rank, out = q.get(timeout=240)
        res[rank] = out
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    for g in range(3):
        f = [lv["f"] for lv in ref["groups"][g]["levels"]]
        for k in range(LEN):
            parents = [res[r][g][k][0] for r in range(world)]
            F = 1 if k == 0 else f[k - 1]
            assert sum(parents) == F and max(parents) - min(parents) <= 1   # balanced parent slices
            assert res[0][g][k][1] == res[1][g][k][1] == f[k]               # global level size = oracle f_k
            assert res[0][g][k][2] == 0                                     # rank offsets: exclusive scan
