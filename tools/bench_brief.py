"""One-screen summary of a bench.py JSON line: python tools/bench_brief.py file.json"""
import json
import sys

d = json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
print(f"C5 ms/step {d['ms_per_step']:.2f}  configs/s {d['value']:.3g}  pairs/s {d.get('pairs_evaluated_per_s', 0):.3g}  "
      f"roofline frac {d['roofline']['frac']:.3f} step {d['roofline']['step']['frac']:.3f}  e2e {d['e2e']['value']:.3g}  "
      f"clocks {d['clocks']}")
for k, v in d.get("secondary", {}).items():
    if "ms_per_step" in v:
        print(f"{k:8s} ms {v['ms_per_step']:.3f} step frac {v.get('roofline_frac_step', 0):.3f} levels {v.get('level_ms')}")
    else:
        print(k, v)
ps = d.get("predicted_scaling") or {}
for mode in ("sync", "replay"):
    if mode in ps:
        print(mode, {n: (round(x["T_ms"], 3), round(x.get("efficiency", 1.0), 3)) for n, x in ps[mode].items()})
if "replay_measured_1_ms" in ps:
    print("replay measured N=1 ms", ps["replay_measured_1_ms"])
if "error" in ps:
    print("predicted_scaling error", ps["error"])
