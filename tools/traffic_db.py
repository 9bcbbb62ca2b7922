"""Record ncu-measured DRAM traffic per launch into profiles/traffic.json (read by bench.py's
roofline).  usage: python tools/traffic_db.py REP KEY[,KEY...] [REP KEY[,KEY...] ...]
KEYs ("spec:g<group>:l<level>", level 0-based) name the report's kernels in capture order."""
import csv
import io
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
path = os.path.join(ROOT, "profiles", "traffic.json")
db = json.load(open(path)) if os.path.exists(path) else {}
args = sys.argv[1:]
for rep, keys in zip(args[::2], args[1::2]):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    h, u = rows[0], rows[1]
    for key, r in zip(keys.split(","), rows[2:]):
        d = dict(zip(h, r))

        def val(k):
            v = float(d[k].replace(",", ""))
            unit = u[h.index(k)]
            return v * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(unit, 1)
        rd, wr = val("dram__bytes_read.sum"), val("dram__bytes_write.sum")
        db[key] = {"dram_bytes": int(rd + wr), "read": int(rd), "write": int(wr), "kernel": d["Kernel Name"],
                   "ncu_us": float(d["gpu__time_duration.sum"].replace(",", "")) *
                   (1e3 if u[h.index("gpu__time_duration.sum")] == "ms" else 1),
                   "source": os.path.basename(rep) + " (ncu --set full --clock-control none)"}
        print(key, db[key])
json.dump(db, open(path, "w"), indent=1, sort_keys=True)
