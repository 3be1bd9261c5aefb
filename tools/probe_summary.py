"""Aggregate a MIMOSE_PROBE_DUMP CSV (M, N, K, epi, us per in-step GEMM launch,
CUDA events on the launching stream) by (N, K, epi): launches, share of the
GEMM time, mean M, achieved TFLOP/s.  Grouped weight-gradient launches are
(T, N1 K1 + N2 K2, tile width, -1).

usage: python tools/probe_summary.py probe.csv [peak_tflops]   (default: MEASURED_PEAKS.json bf16_tflops)
"""
import collections
import json
import os
import sys

EPI = {0: "store", 1: "bias", 2: "bias+gelu", 3: "bias+drop+res", 4: "gelu'", 5: "acc+res f32", 6: "f32",
       8: "bias+gelu_tanh", 9: "gelu_tanh'", 10: "bias+drop+res f32", 11: "acc f32", -1: "grouped wgrad"}

rows = [tuple(float(x) for x in ln.split(",")) for ln in open(sys.argv[1]) if ln.strip()]
_mp = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "MEASURED_PEAKS.json")
peak = float(sys.argv[2]) if len(sys.argv) > 2 else (json.load(open(_mp))["bf16_tflops"] if os.path.exists(_mp) else 1650.0)
agg = collections.defaultdict(lambda: [0, 0.0, 0.0, 0.0])   # n, us, flops, sum M
for M, N, K, e, us in rows:
    key = (int(N), int(K), int(e))
    fl = 2.0 * M * N if e == -1 else 2.0 * M * N * K
    a = agg[key]
    a[0] += 1; a[1] += us; a[2] += fl; a[3] += M
T = sum(a[1] for a in agg.values())
F = sum(a[2] for a in agg.values())
print(f"# {sys.argv[1]}: {len(rows)} launches, {T / 1000:.2f} ms, {F / T / 1e6:.1f} TFLOP/s = {F / T / 1e6 / peak:.3f} of {peak}")
print(f"{'share':>6} {'n':>5} {'mean_us':>8} {'mean_M':>7} {'N':>7} {'K':>6} {'TFLOP/s':>8} {'frac':>5}  epilogue")
for (N, K, e), (n, us, fl, sm) in sorted(agg.items(), key=lambda x: -x[1][1]):
    tf = fl / us / 1e6
    print(f"{100 * us / T:5.1f}% {n:5d} {us / n:8.2f} {sm / n:7.0f} {N:7d} {K:6d} {tf:8.1f} {tf / peak:5.2f}  {EPI.get(e, e)}")
