"""the CPU oracle timed on this host (run on the GPU box, same job as the bench).

For every config: O2 (pruned nested loop, interpreted bytecode) generation time at 1 thread and
at all hardware threads, median of 3 (oracle's own steady clock, spec parsing excluded); O1
(literal full-product brute force) on C1; C5 on a bounded sample (rates, and the full-size time
extrapolated from the evals rate); C4 as the oracle's decode of 10^6 indices.  Writes one JSON
object to stdout.   python tools/cpu_baselines.py > gpurun_out/cpu_baselines.json
"""
import json
import os
import statistics
import subprocess
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import atfspec as A  # noqa: E402
from atfspec.fuzz import splitmix64_indices  # noqa: E402
from oracle import run as orc  # noqa: E402


def lscpu_model():
    try:
        out = subprocess.run(["lscpu"], capture_output=True, text=True).stdout
        for line in out.splitlines():
            if line.lower().startswith("model name"):
                return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return None


def o2(spec, threads, reps=3):
    ts, d = [], None
    for _ in range(reps):
        d = orc.info(spec, threads=threads)
        ts.append(d["gen_seconds"])
    evals = sum(lv["evals"] for g in d["groups"] for lv in g["levels"])
    leaves = sum(g["size"] for g in d["groups"])
    t = statistics.median(ts)
    return {"threads": threads, "median_s": t, "runs_s": ts, "evals": evals, "group_leaves": leaves,
            "S": d["S"], "configs_per_s": leaves / t if t else None, "evals_per_s": evals / t if t else None}


def main():
    orc.build()
    cores = os.cpu_count() or 1
    res = {"host": {"lscpu_model": lscpu_model(), "nproc": cores}, "configs": {}}
    specs = {"C1": A.c1_toy(), "C2": A.c2_xgemm_direct(256), "C3-IS1": A.c3_xgemm("IS1"),
             "C3-IS3": A.c3_xgemm("IS3"), "C3-IS2": A.c3_xgemm("IS2"), "C3-IS4": A.c3_xgemm("IS4")}
    for name, spec in specs.items():
        t0 = time.time()
        r = {"O2_1thread": o2(spec, 1), f"O2_{cores}threads": o2(spec, cores)}
        if name == "C1":
            o1 = [orc.o1(spec)[0] for _ in range(3)]
            r["O1_1thread"] = {"median_s": statistics.median(x["seconds"] for x in o1), "evaluated": o1[0]["evaluated"]}
        r["wall_s"] = time.time() - t0
        res["configs"][name] = r
        print(name, json.dumps(r)[:200], file=sys.stderr, flush=True)
    # C5: bounded sample (the full O2 run is ~10^11 interpreted evaluations)
    spec = A.c5_chains(4096, 8)
    total_evals = 171147067392
    c5 = {}
    for th in (1, cores):
        d = orc.time_sample(spec, threads=th, budget_s=20.0, timeout=600)
        rate = d["evals"] / d["seconds"]
        c5[f"{th}threads"] = {"sample_s": d["seconds"], "evals": d["evals"], "leaves": d["leaves"],
                              "evals_per_s": rate, "configs_per_s": d["leaves"] / d["seconds"],
                              "extrapolated_full_s": total_evals / rate}
    res["configs"]["C5"] = c5
    # C4: oracle decode of 10^6 of the 10^8 indices (each call regenerates the group)
    spec = A.c3_xgemm("IS2")
    S = 1692310928
    idx = splitmix64_indices(1_000_000, S, A.c4_indices_seed())
    ts = []
    for _ in range(3):
        t0 = time.time()
        orc.decode(spec, idx, threads=cores, want_rows=False)
        ts.append(time.time() - t0)
    res["configs"]["C4-decode-1e6"] = {"threads": cores, "median_s": statistics.median(ts), "runs_s": ts,
                                       "note": "wall time of the oracle's decode command (regenerates C3-IS2's "
                                               "group 0 with O2, then picks the 10^6 digits)"}
    print(json.dumps(res))


if __name__ == "__main__":
    main()
