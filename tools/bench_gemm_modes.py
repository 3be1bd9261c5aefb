"""Mainloop-only GEMM timing (EPI_NONE) across kernel variants, BERT-base shapes."""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_liaolysshfyctzlq23_b200 import binding as mb  # noqa: E402
from tools.bench_gemm import timeit  # noqa: E402

T = int(sys.argv[1]) if len(sys.argv) > 1 else 5120
H, F = 768, 3072
bf = torch.bfloat16
A = torch.randn(max(T, F), max(F, T), device="cuda", dtype=bf)
B = torch.randn(max(T, F), max(F, T), device="cuda", dtype=bf)
C = torch.empty(16, device="cuda")
shapes = [("NT T x 3072 x 768", T, F, H, H, 1, H, 1), ("NT T x 768 x 3072", T, H, F, F, 1, F, 1),
          ("NT T x 2304 x 768", T, 3 * H, H, H, 1, H, 1), ("TN 3072 x 768 x T", F, H, T, 1, F, 1, H),
          ("NN T x 3072 x 768", T, F, H, H, 1, 1, F)]
for name, M, N, K, asm, ask, bsn, bsk in shapes:
    fl = 2.0 * M * N * K
    for mode in [int(x) for x in os.environ.get("MODES", "0,11,12,21,22").split(",")]:
        mb.debug_options(gemm_mode=mode)
        us = timeit(lambda: mb.debug_gemm_ex(7, M, N, K, A, asm, ask, B, bsn, bsk, C, N))
        print(f"{name:20s} mode={mode:2d} {us:8.1f} us {fl / us / 1e6:7.1f} TFLOP/s", flush=True)
mb.debug_options(gemm_mode=2)
