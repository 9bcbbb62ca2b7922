"""Summarise an ncu --metrics gpu__time_duration.sum launch list (CSV) per kernel."""
import csv
import sys


def load(path):
    rows = list(csv.reader(open(path)))
    hdr, out = None, []
    for r in rows:
        if r and r[0] == "ID":
            hdr = r
            continue
        if hdr and len(r) == len(hdr):
            d = dict(zip(hdr, r))
            if d["Metric Name"] == "gpu__time_duration.sum":
                v = float(d["Metric Value"].replace(",", ""))
                if d["Metric Unit"] == "us":
                    v *= 1e3
                elif d["Metric Unit"] == "ms":
                    v *= 1e6
                out.append((d["Kernel Name"], v))
    return out


if __name__ == "__main__":
    out = load(sys.argv[1])
    tot = sum(v for _, v in out)
    for k, v in out:
        print(f"{v/1e3:12.1f} us  {100*v/tot:5.1f}%  {k[:60]}")
    print(f"total {tot/1e6:.3f} ms over {len(out)} launches")
