"""Opcode census of the wide kernel's unrolled hot loop (from the first LDS.128 of the table
to the queue ballot) for every expand_wide instantiation: python tools/sass_hot.py file.o"""
import re
import subprocess
import sys

obj = sys.argv[1]
sass = subprocess.run(["cuobjdump", "-sass", obj], capture_output=True, text=True).stdout
for f in re.split(r"\n\s*Function : ", sass)[1:]:
    name = f.split("\n", 1)[0].strip()
    if "expand_wide" not in name and "expand_wtile" not in name:
        continue
    L = [re.sub(r"/\* 0x[0-9a-f]+ \*/", "", l) for l in f.split("\n") if l.strip().startswith("/*")]
    # densest window of VIMNMX3 = the unrolled body
    idx = [i for i, l in enumerate(L) if "VIMNMX3" in l]
    if not idx:
        print(f"{name[:48]:48s} no hot loop")
        continue
    best = None
    for a in idx:
        b = a
        while b + 1 < len(L) and (b + 1 - a) < 400:
            b += 1
            if "VOTE" in L[b] or "BRA" in L[b]:
                break
        n3 = sum("VIMNMX3" in L[k] for k in range(a, b + 1))
        if best is None or n3 > best[2]:
            best = (a, b, n3)
    a, b, _ = best
    cnt = {}
    for l in L[a - 20:b + 1]:
        m = re.search(r"\*/\s+(?:@!?U?P\w+\s+)?([A-Z][A-Z0-9_]*)", l)
        if m:
            cnt[m.group(1)] = cnt.get(m.group(1), 0) + 1
    top = sorted(cnt.items(), key=lambda x: -x[1])[:9]
    print(f"{name[:48]:48s} " + " ".join(f"{k}:{v}" for k, v in top))
