"""Critical-path prediction of the steady-state (replay) balanced generation vs the lock-step one.

In the replay protocol a rank waits only on the device flags of the ranks that own its next parent
slice, not on every rank: with groups on rank subsets (the default; plain partition:
ATF_FLAG_DIST_NO_SUBSETS) the
groups' rank sets progress independently.  From the per-rank per-round device times of N virtual
ranks (one rank's round alone on the GPU, ATF_FLAG_TIMING), this prints
  lockstep: sum over rounds of the slowest rank's round (the bench's "replay" model), and
  critical: end[r][k] = max(end[r][k-1], max over q sharing a group with r of end[q][k-1] + flag)
            + dur[r][k]  (conservative: every rank of a shared group counts as an owner),
for the plain partition and for subsets.   python tools/dist_critical.py [N ...]"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import atfspec as A  # noqa: E402
from paper_conf_hpdc_raschg18_b200 import Space, _lib as L  # noqa: E402
from paper_conf_hpdc_raschg18_b200.shard import virtual_ranks  # noqa: E402

FLAG_US = 10.0
AG_US = 25.0


def predict(spec, N, subsets, reps=3):
    flags = L.ATF_FLAG_NO_SEG_BOUNDS | L.ATF_FLAG_TIMING | (0 if subsets else L.ATF_FLAG_DIST_NO_SUBSETS)
    spaces = [Space(spec, flags=flags) for _ in range(N)]
    try:
        for _ in range(2):          # first generation: plain partition; subsets from the second on
            virtual_ranks(spaces)
        G = spaces[0].num_groups()
        best = None
        for _ in range(reps):
            torch.cuda.synchronize()
            virtual_ranks(spaces, serialize=True)
            dur = [[x * 1e-3 for x in sp.dist_round_ms()] for sp in spaces]
            R = len(dur[0])
            member = [[any(sp.level_view(g, k)["n_nodes"] > 0 for k in range(sp.num_levels(g))) for g in range(G)]
                      for sp in spaces]
            deps = [[q for q in range(N) if any(member[r][g] and member[q][g] for g in range(G))] for r in range(N)]
            lock = sum(max(dur[r][k] for r in range(N)) for k in range(R))
            end = [0.0] * N
            for k in range(R):
                new = []
                for r in range(N):
                    start = end[r]
                    if k:
                        start = max(start, max(end[q] for q in deps[r] if q != r) + FLAG_US * 1e-6
                                    if len(deps[r]) > 1 else start)
                    new.append(start + dur[r][k])
                end = new
            crit = max(end)
            cand = (crit, lock, [sum(d) for d in dur], [[g for g in range(G) if member[r][g]] for r in range(N)])
            if best is None or cand[0] < best[0]:
                best = cand
        return {"critical_ms": round((best[0] + AG_US * 1e-6) * 1e3, 3),
                "lockstep_ms": round((best[1] + AG_US * 1e-6) * 1e3, 3),
                "rank_busy_ms": [round(x * 1e3, 3) for x in best[2]], "groups": best[3]}
    finally:
        for sp in spaces:
            sp.close()


def main():
    worlds = [int(x) for x in sys.argv[1:]] or [1, 2, 4, 8]
    spec = A.c5_chains(4096, 8)
    out = {}
    for subsets in (False, True):
        for N in worlds:
            if subsets and N == 1:
                continue
            res = predict(spec, N, subsets)
            out[f"{'subsets' if subsets else 'plain'}_{N}"] = res
            print(N, "subsets" if subsets else "plain", res, flush=True)
    t1 = out.get("plain_1", {}).get("critical_ms")
    if t1:
        for k, v in out.items():
            n = int(k.split("_")[1])
            v["eff_critical"] = round(t1 / (n * v["critical_ms"]), 3)
            v["eff_lockstep"] = round(t1 / (n * v["lockstep_ms"]), 3)
    print(json.dumps(out))


if __name__ == "__main__":
    main()
