"""One mainloop-only (EPI_NONE) GEMM launch in a given mode, for ncu:
    python tools/probe_modes.py MODE M N K [a_mn b_mn]"""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_liaolysshfyctzlq23_b200 import binding as mb  # noqa: E402
from tools.bench_gemm import timeit  # noqa: E402

mode, M, N, K = (int(v) for v in sys.argv[1:5])
a_mn, b_mn = (int(v) for v in sys.argv[5:7]) if len(sys.argv) > 6 else (0, 0)
A = torch.randn(M * K, device="cuda").bfloat16()
B = torch.randn(N * K, device="cuda").bfloat16()
C = torch.empty(16, device="cuda")
asm, ask = (1, M) if a_mn else (K, 1)
bsn, bsk = (1, N) if b_mn else (K, 1)
mb.debug_options(gemm_mode=mode)
us = timeit(lambda: mb.debug_gemm_ex(7, M, N, K, A, asm, ask, B, bsn, bsk, C, N))
print(f"mode={mode} {M}x{N}x{K} a_mn={a_mn} b_mn={b_mn}: {us:.1f} us {2.0 * M * N * K / us / 1e6:.1f} TFLOP/s")
