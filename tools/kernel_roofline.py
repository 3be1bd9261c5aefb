"""Per-kernel-class time share and achieved DRAM bandwidth from an ncu metrics CSV.

    ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum \\
        --clock-control none --csv --log-file gpurun_out/kern.csv python bench.py ...
    python tools/kernel_roofline.py gpurun_out/kern.csv [hbm_gbs]

ncu replays each launch with a flushed L2 and serialised: shares and GB/s are
cold-cache figures (an upper bound on traffic, a lower bound on bandwidth of
the warm step)."""
import collections
import csv
import re
import sys

UNIT = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "ns": 1e-9, "us": 1e-6, "usecond": 1e-6,
        "nsecond": 1e-9, "msecond": 1e-3, "ms": 1e-3}


def main(src, peak):
    lines = [l for l in open(src) if l.startswith('"')]
    per = collections.defaultdict(dict)
    names = {}
    for r in csv.DictReader(lines):
        names[r["ID"]] = re.sub(r"\(.*", "", r["Kernel Name"])[:56]
        per[r["ID"]][r["Metric Name"]] = float(r["Metric Value"].replace(",", "")) * UNIT.get(r["Metric Unit"], 1.0)
    agg = collections.defaultdict(lambda: [0, 0.0, 0.0])
    for k, m in per.items():
        a = agg[names[k]]
        a[0] += 1
        a[1] += m.get("gpu__time_duration.sum", 0.0)
        a[2] += m.get("dram__bytes_read.sum", 0.0) + m.get("dram__bytes_write.sum", 0.0)
    T = sum(a[1] for a in agg.values())
    print(f"# {src}: {sum(a[0] for a in agg.values())} launches, {T * 1e3:.1f} ms (cold-cache, serialised); "
          f"HBM peak {peak:.0f} GB/s (MEASURED_PEAKS.json hbm_gbs)")
    print(f"{'share':>7} {'n':>5} {'avg_us':>8} {'MB/launch':>10} {'GB/s':>7} {'of_hbm':>7}  kernel")
    for name, (n, t, b) in sorted(agg.items(), key=lambda x: -x[1][1]):
        gbs = b / t / 1e9 if t else 0.0
        print(f"{100 * t / T:6.2f}% {n:5d} {t / n * 1e6:8.2f} {b / n / 1e6:10.2f} {gbs:7.0f} {gbs / peak:7.2f}  {name}")


if __name__ == "__main__":
    main(sys.argv[1], float(sys.argv[2]) if len(sys.argv) > 2 else 6452.2)
