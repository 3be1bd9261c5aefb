"""GEMM microbenchmark: the BERT-base step's GEMM shapes (T tokens) through the
library's kernels in every mode, against cuBLAS (torch.matmul) for the plain
product.  Prints one line per (shape, epilogue, mode): us, TFLOP/s."""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_liaolysshfyctzlq23_b200 import binding as mb  # noqa: E402


def timeit(fn, reps=20):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(reps):
        fn()
    b.record()
    torch.cuda.synchronize()
    return a.elapsed_time(b) / reps * 1000.0


def main():
    T = int(sys.argv[1]) if len(sys.argv) > 1 else 5120
    only = sys.argv[2] if len(sys.argv) > 2 else ""          # substring filter on the case name
    modes = [int(m) for m in sys.argv[3].split(",")] if len(sys.argv) > 3 else [1, 12]
    H, F = 768, 3072
    dev = "cuda"
    bf = torch.bfloat16
    x = torch.randn(T, H, device=dev, dtype=bf)
    h1 = torch.randn(T, H, device=dev, dtype=bf)
    g = torch.randn(T, F, device=dev, dtype=bf)
    u = torch.randn(T, F, device=dev, dtype=bf)
    wq = torch.randn(3 * H, H, device=dev, dtype=bf)
    wo = torch.randn(H, H, device=dev, dtype=bf)
    w1 = torch.randn(F, H, device=dev, dtype=bf)
    w2 = torch.randn(H, F, device=dev, dtype=bf)
    bias = torch.randn(max(3 * H, F), device=dev, dtype=bf)
    dy3 = torch.randn(T, 3 * H, device=dev, dtype=bf)
    dyF = torch.randn(T, F, device=dev, dtype=bf)
    dyH = torch.randn(T, H, device=dev, dtype=bf)
    outb = torch.empty(T, max(3 * H, F), device=dev, dtype=bf)
    outb2 = torch.empty(T, F, device=dev, dtype=bf)
    outf = torch.empty(T, max(3 * H, F), device=dev)
    resf = torch.randn(T, H, device=dev)
    ws = torch.empty(4 * F * H, device=dev)
    cases = [
        # name, epi, M, N, K, A, a_sm, a_sk, B, b_sn, b_sk, extra
        ("fwd QKV  bias", 1, T, 3 * H, H, x, H, 1, wq, H, 1, {}),
        ("fwd out  drop+res", 3, T, H, H, x, H, 1, wo, H, 1, dict(res=x, ldr=H)),
        ("fwd FFN1 gelu", 2, T, F, H, h1, H, 1, w1, H, 1, dict(C2=outb2)),
        ("fwd FFN2 drop+res", 3, T, H, F, g, F, 1, w2, F, 1, dict(res=h1, ldr=H)),
        ("dgr FFN2 gelu'", 4, T, F, H, dyH, H, 1, w2, 1, F, dict(aux=u, ldx=F)),
        ("dgr FFN1 +res", 5, T, H, F, dyF, F, 1, w1, 1, H, dict(res=resf, ldr=H)),
        ("dgr QKV  +res", 5, T, H, 3 * H, dy3, 3 * H, 1, wq, 1, H, dict(res=resf, ldr=H)),
        ("dgr out  store", 0, T, H, H, dyH, H, 1, wo, 1, H, {}),
        ("wgr FFN2 (H,F,T)", 6, H, F, T, dyH, 1, H, g, 1, F, {}),
        ("wgr FFN1 (F,H,T)", 6, F, H, T, dyF, 1, F, h1, 1, H, {}),
        ("wgr QKV (3H,H,T)", 6, 3 * H, H, T, dy3, 1, 3 * H, x, 1, H, {}),
        ("wgr out  (H,H,T) s4", 6, H, H, T, dyH, 1, H, x, 1, H, dict(split=4)),
    ]
    for name, epi, M, N, K, A, asm, ask, B, bsn, bsk, ex in cases:
        if only and only not in name:
            continue
        fl = 2.0 * M * N * K
        split = ex.pop("split", 1)
        C = (outf if epi in (3, 5, 6) else outb)
        C_ = ws if split > 1 else C
        for mode in modes:
            mb.debug_options(gemm_mode=mode)
            us = timeit(lambda: mb.debug_gemm_ex(epi, M, N, K, A, asm, ask, B, bsn, bsk, C_, N, bias=bias,
                                                 split=split, **ex))
            print(f"{name:22s} T={T:5d} mode={mode}  {us:8.1f} us  {fl / us / 1e6:7.1f} TFLOP/s", flush=True)
        # cuBLAS reference of the plain product (same operand layouts)
        At = A if ask == 1 else A.t()
        Am = At.view(M, K) if ask == 1 else A.t()
        Bm = B if bsk == 1 else B.t()
        us = timeit(lambda: torch.matmul(Am, Bm.t() if bsk == 1 else B))
        print(f"{name:22s} T={T:5d} cuBLAS  {us:8.1f} us  {fl / us / 1e6:7.1f} TFLOP/s", flush=True)
    mb.debug_options(gemm_mode=1)


if __name__ == "__main__":
    main()
