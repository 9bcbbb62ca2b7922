"""Per-level roofline table of one spec (serialized groups, CUDA events per expand kernel):
group, level, kernel, r, parents, children, evals, expand ms, level ms, fraction of the ALU peak.
usage (on a GPU box): python tools/level_frac.py [C5|C3-IS2|...] [steps]"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402

import atfspec as A  # noqa: E402
import bench  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "C5"
steps = int(sys.argv[2]) if len(sys.argv) > 2 else 5
spec = A.config_spec(name)
res = bench.run_generation(spec, steps, 3, timing=True, serial=True)
plan = res["plan"]
lv = [(gi, k, l) for gi, g in enumerate(plan["groups"]) for k, l in enumerate(g["levels"])]
exp_ms = np.array(res["level_exp_ms"], dtype=np.float64).mean(axis=0)
lvl_ms = np.array(res["level_ms"], dtype=np.float64).mean(axis=0)
peak = bench.int_peak_ops(1965.0)
kn = {0: "narrow", 1: "wide", 2: "wtile", 3: "nfast", 4: "nfastJ"}
print(f"{name}: step(serial) {lvl_ms.sum():.3f} ms, expand {exp_ms.sum():.3f} ms")
print(f"{'g':>2} {'lvl':>3} {'kern':>6} {'r':>5} {'parents':>10} {'children':>10} {'evals':>12} "
      f"{'exp_ms':>8} {'lvl_ms':>8} {'frac':>6} {'tested':>6}")
for (g, k, l), s, e, t in zip(lv, res["stats"], exp_ms, lvl_ms):
    ops = (s["pairs"] or s["evals"]) * l["cost"]
    fr = ops / (e * 1e-3) / peak if e > 0 else 0.0
    par = s["evals"] // max(1, s["r"])
    print(f"{g:>2} {k + 1:>3} {kn.get(s.get('kernel', -1), '?'):>6} {s['r']:>5} {par:>10} {s['f']:>10} "
          f"{s['evals']:>12} {e:>8.3f} {t:>8.3f} {fr:>6.3f} {(s['pairs'] or s['evals']) / max(1, s['evals']):>6.3f}")
