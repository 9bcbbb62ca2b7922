"""Per-CUDA-line warp-stall samples and executed instructions from an ncu report
(--page source --print-source cuda,sass): python tools/ncu_source.py rep [top] [kernel-name]
[--skip=N] (the N-th launch of that kernel only) [--src=file] (source text for the line numbers,
e.g. an NVRTC source written by tools/dump_jit.py) [--by-inst]"""
import csv
import io
import subprocess
import sys

pos = [a for a in sys.argv[1:] if not a.startswith("--")]
opt = dict(a[2:].split("=", 1) for a in sys.argv[1:] if a.startswith("--") and "=" in a)
rep = pos[0]
top = int(pos[1]) if len(pos) > 1 else 25
kfilter = ["-k", pos[2]] if len(pos) > 2 else []
if "skip" in opt:
    kfilter += ["--launch-skip", opt["skip"], "--launch-count", "1"]
local = open(opt["src"]).read().split("\n") if "src" in opt else None
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"] + kfilter,
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
agg, src, fname = {}, {}, None
hdr = None
for r in rows:
    if len(r) == 2 and r[0] == "File Path":
        fname = r[1].split("/")[-1]
        continue
    if r and r[0] == "Line No":
        hdr = r
        continue
    if hdr is None or len(r) != len(hdr) or not r[0].strip():
        continue
    key = (fname, int(r[0]))
    src[key] = local[int(r[0]) - 1] if local and 0 < int(r[0]) <= len(local) else r[1]
    s = float(r[4] or 0)
    ins = float(r[7] or 0)
    a = agg.setdefault(key, [0.0, 0.0])
    a[0] += s
    a[1] += ins
tot_s = sum(v[0] for v in agg.values()) or 1
tot_i = sum(v[1] for v in agg.values()) or 1
print(f"total stall samples {tot_s:.0f}, warp instructions {tot_i:.3g}")
order = 1 if "--by-inst" in sys.argv else 0
for k, v in sorted(agg.items(), key=lambda kv: -kv[1][order])[:top]:
    print(f"{k[0]:>16}:{k[1]:<5d} stall {100*v[0]/tot_s:5.1f}%  inst {100*v[1]/tot_i:5.1f}%  {src[k].strip()[:80]}")
