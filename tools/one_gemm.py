"""Run one library GEMM (EPI given) a few times: for ncu captures of a single variant.
    python tools/one_gemm.py MODE EPI M N K [a_mn b_mn] [reps]"""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_liaolysshfyctzlq23_b200 import binding as mb  # noqa: E402
from tools.bench_gemm import timeit  # noqa: E402

mode, epi, M, N, K = (int(x) for x in sys.argv[1:6])
a_mn = int(sys.argv[6]) if len(sys.argv) > 6 else 0
b_mn = int(sys.argv[7]) if len(sys.argv) > 7 else 0
reps = int(sys.argv[8]) if len(sys.argv) > 8 else 20
bf = torch.bfloat16
A = torch.randn(K, M, device="cuda", dtype=bf) if a_mn else torch.randn(M, K, device="cuda", dtype=bf)
B = torch.randn(K, N, device="cuda", dtype=bf) if b_mn else torch.randn(N, K, device="cuda", dtype=bf)
a_sm, a_sk = (1, M) if a_mn else (K, 1)
b_sn, b_sk = (1, N) if b_mn else (K, 1)
C = torch.empty(M, N, device="cuda")
C2 = torch.empty(M, N, device="cuda", dtype=bf)
bias = torch.randn(N, device="cuda", dtype=bf)
res = torch.randn(M, N, device="cuda", dtype=bf)
kw = dict(bias=bias)
if epi == 2:
    kw["C2"] = C2
if epi in (3,):
    kw.update(res=res, ldr=N)
if epi == 4:
    kw.update(aux=res, ldx=N)
if epi == 5:
    kw.update(res=C, ldr=N)
mb.debug_options(gemm_mode=mode)
us = timeit(lambda: mb.debug_gemm_ex(epi, M, N, K, A, a_sm, a_sk, B, b_sn, b_sk, C, N, **kw), reps=reps)
print(f"mode={mode} epi={epi} {M}x{N}x{K} a_mn={a_mn} b_mn={b_mn}: {us:.1f} us {2.0 * M * N * K / us / 1e6:.1f} TFLOP/s")
