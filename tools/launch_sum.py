"""Summarise an ncu launch list (--metrics gpu__time_duration.sum --csv): the last half of the
launches (gen_once.py --reps 2 profiles two generations), launches above a threshold.
python tools/launch_sum.py launches.csv [min_us]"""
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
thr = float(sys.argv[2]) if len(sys.argv) > 2 else 20.0
hdr, out = None, []
for r in rows:
    if "Kernel Name" in r:
        hdr = r
        continue
    if hdr and len(r) == len(hdr):
        d = dict(zip(hdr, r))
        if d.get("Metric Name") == "gpu__time_duration.sum":
            v = float(d["Metric Value"]) / (1000.0 if d.get("Metric Unit") in ("ns", "nsecond") else 1.0)
            out.append((d["ID"], d["Kernel Name"][:60], v))
n = len(out) // 2
print(f"{n} launches per generation, total {sum(x[2] for x in out[n:]):.1f} us")
for x in out[n:]:
    if x[2] >= thr:
        print(f"  {x[0]:>5} {x[2]:9.1f} us  {x[1]}")
