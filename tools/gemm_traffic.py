"""Per-launch DRAM traffic of the GEMM kernels from an ncu metrics CSV.

    ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum \\
        -k regex:k_gemm_tc --csv --log-file gpurun_out/gemm_dram.csv \\
        python bench.py --steps 3 --warmup 3 --no-baselines --no-cpu-baseline
    python tools/gemm_traffic.py gpurun_out/gemm_dram.csv profiles/r1/gemm_traffic.json
"""
import csv
import json
import sys
from collections import defaultdict

UNIT = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "KB": 1e3, "MB": 1e6, "GB": 1e9,
        "ns": 1e-9, "us": 1e-6, "usecond": 1e-6, "nsecond": 1e-9, "msecond": 1e-3}


def main(src, dst):
    lines = [l for l in open(src) if l.startswith('"')]
    rows = list(csv.DictReader(lines))
    per = defaultdict(dict)
    names = {}
    for r in rows:
        k = r["ID"]
        names[k] = r["Kernel Name"]
        v = float(r["Metric Value"].replace(",", "")) * UNIT.get(r["Metric Unit"], 1.0)
        per[k][r["Metric Name"]] = v
    launches = [m for k, m in per.items() if "dram__bytes_read.sum" in m and "k_gemm_tc" in names[k]]
    rd = sum(m["dram__bytes_read.sum"] for m in launches)
    wr = sum(m.get("dram__bytes_write.sum", 0.0) for m in launches)
    t = sum(m.get("gpu__time_duration.sum", 0.0) for m in launches)
    n = len(launches)
    out = {"launches": n, "dram_bytes_per_launch": (rd + wr) / max(n, 1),
           "dram_read_bytes_per_launch": rd / max(n, 1), "dram_write_bytes_per_launch": wr / max(n, 1),
           "mean_duration_us": 1e6 * t / max(n, 1),
           "how": "ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum over every k_gemm_tc* launch of "
                  "`bench.py --steps 2 --warmup 3 --no-baselines --no-cpu-baseline` (cold cache per launch, "
                  "ncu default cache control)",
           "source": src}
    json.dump(out, open(dst, "w"), indent=1)
    print(json.dumps(out))


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2])
