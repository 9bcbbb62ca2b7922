"""Write the oracle's expected values for the full-size configs to tests/golden/*.json.

Calls only oracle/ (and atfspec to build the input specs).  Run from the repo root:
    python tests/golden/make_golden.py [--threads 8] [--only NAME ...]
Every stored value is the C++ oracle's output (O2 per group), never the CUDA path's.
"""
import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import atfspec as A  # noqa: E402
from atfspec.fuzz import splitmix64_indices  # noqa: E402
from oracle import run as orc  # noqa: E402

HERE = os.path.dirname(os.path.abspath(__file__))

SPECS = {
    "C1": A.c1_toy,
    "C2": lambda: A.c2_xgemm_direct(256),
    "C2-1024": lambda: A.c2_xgemm_direct(1024),
    "C3-IS1": lambda: A.c3_xgemm("IS1"),
    "C3-IS2": lambda: A.c3_xgemm("IS2"),
    "C3-IS3": lambda: A.c3_xgemm("IS3"),
    "C3-IS4": lambda: A.c3_xgemm("IS4"),
    "C3-IS4-anchored": lambda: A.c3_xgemm("IS4", anchored=True),
    "C5-512": lambda: A.c5_chains(512, 8),
    # configs[4] at full size (the bench workload): per-group leaf hashes + element-wise windows
    "C5": lambda: A.c5_chains(4096, 8),
}

# element-wise windows of leaf rows (first / middle / last WINDOW leaves of every group), from
# the oracle's canonical leaf stream (oracle/atf_oracle leaves)
WINDOW = 1024
WINDOWS = {"C5", "C5-512"}

# decode samples: (spec name, number of splitmix indices)
DECODES = {
    "C3-IS2": 1_000_000,
    "C3-IS4": 1_000_000,
}
# C4 (configs[3]) in full: the order-dependent hash of ALL 10^8 decoded rows (oracle decode
# streams every group once and picks the requested digits; rows are not stored)
DECODES_FULL = {
    "C3-IS2": 100_000_000,
}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--threads", type=int, default=os.cpu_count())
    ap.add_argument("--only", nargs="*")
    a = ap.parse_args()
    for name, mk in SPECS.items():
        if a.only and name not in a.only:
            continue
        t0 = time.time()
        spec = mk()
        d = orc.info(spec, threads=a.threads, hash=True)
        d["spec_name"] = name
        d["generated_by"] = "tests/golden/make_golden.py -> oracle/atf_oracle info --hash"
        if name in DECODES:
            n = DECODES[name]
            S = int(d["S"])
            idx = splitmix64_indices(n, S, A.c4_indices_seed())
            dec, soa = orc.decode(spec, idx, threads=a.threads, want_rows=True)
            d["decode"] = {"n": n, "seed": A.c4_indices_seed(), "hash": dec["hash"],
                           "first_rows": soa[:, :8].T.tolist(),
                           "recipe": "idx_i = splitmix64(seed + i) mod S"}
        if name in DECODES_FULL:
            n = DECODES_FULL[name]
            S = int(d["S"])
            idx = splitmix64_indices(n, S, A.c4_indices_seed())
            dec, _ = orc.decode(spec, idx, threads=a.threads, want_rows=False)
            d["decode_full"] = {"n": n, "seed": A.c4_indices_seed(), "hash": dec["hash"],
                                "recipe": "idx_i = splitmix64(seed + i) mod S, i < n; hash over all n rows"}
            del idx
        if name in WINDOWS:
            d["windows"] = []
            for g, grp in enumerate(d["groups"]):
                lv = orc.leaves(spec, g, len(grp["members"]))
                assert lv.shape[0] == grp["size"]
                n = lv.shape[0]
                starts = sorted({0, max(0, n // 2 - WINDOW // 2), max(0, n - WINDOW)})
                d["windows"].append([{"start": s0, "rows": lv[s0:s0 + WINDOW].tolist()} for s0 in starts])
                del lv
        with open(os.path.join(HERE, f"{name}.json"), "w") as f:
            json.dump(d, f, indent=None if name in WINDOWS else 1)
        print(f"{name}: S={d['S']} ({time.time() - t0:.1f}s)", flush=True)


if __name__ == "__main__":
    main()
