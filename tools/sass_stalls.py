"""Per-instruction stall table from `ncu --page source --csv --print-source=sass`:
prints instructions with >= MIN samples and their dominant stall reasons, plus
totals per contiguous region.   python tools/sass_stalls.py file.csv [MIN] [lo hi]"""
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
h = rows[1]
data = rows[2:]
mn = int(sys.argv[2]) if len(sys.argv) > 2 else 10
lo, hi = (int(sys.argv[3]), int(sys.argv[4])) if len(sys.argv) > 4 else (0, len(data))
isrc = h.index("Source")
iall = h.index("Warp Stall Sampling (All Samples)")
iex = h.index("Instructions Executed")
reasons = [i for i, k in enumerate(h) if k.startswith("stall_") and "Not Issued" not in k]
num = lambda s: float(s) if s not in ("", "-") else 0.0
tot = sum(num(r[iall]) for r in data)
print("total samples", tot)
for i in range(lo, min(hi, len(data))):
    r = data[i]
    s = num(r[iall])
    if s >= mn:
        top = sorted(((num(r[j]), h[j][6:]) for j in reasons), reverse=True)[:3]
        print(f"{i:5d} {int(s):5d} ex={r[iex]:>8s} {r[isrc].strip()[:70]:70s} " +
              " ".join(f"{k}={int(v)}" for v, k in top if v > 0))
