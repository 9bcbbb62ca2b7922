"""Opcode census of the wide kernel's hot loop (the VIMNMX3 min-reduction region)
for every expand_wide instantiation in an object file: python tools/sass_hot.py file.o"""
import re
import subprocess
import sys

obj = sys.argv[1]
sass = subprocess.run(["cuobjdump", "-sass", obj], capture_output=True, text=True).stdout
funcs = re.split(r"\n\s*Function : ", sass)
for f in funcs[1:]:
    name = f.split("\n", 1)[0].strip()
    if "expand_wide" not in name:
        continue
    L = [re.sub(r"/\* 0x[0-9a-f]+ \*/", "", l) for l in f.split("\n")]
    idx = [i for i, l in enumerate(L) if re.search(r"VIMNMX3", l)]
    if not idx:
        print(name, "no hot loop")
        continue
    seg = L[min(idx) - 12:max(idx) + 12]
    cnt = {}
    for l in seg:
        m = re.search(r"\*/\s+(?:@!?U?P\w+\s+)?([A-Z][A-Z0-9_]*)", l)
        if m:
            cnt[m.group(1)] = cnt.get(m.group(1), 0) + 1
    top = sorted(cnt.items(), key=lambda x: -x[1])[:8]
    print(f"{name[:45]:45s} or={len(idx):3d} " + " ".join(f"{k}:{v}" for k, v in top))
