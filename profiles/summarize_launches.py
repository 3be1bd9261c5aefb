"""Aggregate an ncu launch list (gpu__time_duration.sum CSV) by kernel name."""
import collections
import csv
import re
import sys

rows = list(csv.reader(open(sys.argv[1])))
hi = [i for i, r in enumerate(rows) if "Kernel Name" in r][0]
h, data = rows[hi], rows[hi + 1:]
ki, vi, ui = h.index("Kernel Name"), h.index("Metric Value"), h.index("Metric Unit")
scale = {"ns": 1e-3, "us": 1.0, "ms": 1e3}
tot, cnt = collections.defaultdict(float), collections.Counter()
for r in data:
    if len(r) <= vi:
        continue
    v = float(r[vi].replace(",", "")) * scale[r[ui]]
    k = re.sub(r"\(.*", "", r[ki])[:64]
    tot[k] += v
    cnt[k] += 1
T = sum(tot.values())
print(f"# {sys.argv[1]}: {sum(cnt.values())} launches, {T/1000:.1f} ms total (cold-cache, serialised)")
print(f"{'share':>7} {'total_us':>10} {'n':>6} {'avg_us':>8}  kernel")
for k, v in sorted(tot.items(), key=lambda x: -x[1])[:int(sys.argv[2]) if len(sys.argv) > 2 else 30]:
    print(f"{100*v/T:6.2f}% {v:10.1f} {cnt[k]:6d} {v/cnt[k]:8.2f}  {k}")
