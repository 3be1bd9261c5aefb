# GEMM microbenchmark: step shapes at BERT-base T, and large square shapes (steady-state mainloop rate)
python tools/bench_gemm.py 5376 "" 1
for s in 4096 8192; do python tools/one_gemm.py 1 0 $s $s $s 0 0 10; python tools/one_gemm.py 12 0 $s $s $s 0 0 10; done
python - <<'PY'
import torch
from tools.bench_gemm import timeit
for s in (4096, 8192):
    a = torch.randn(s, s, device="cuda", dtype=torch.bfloat16); b = torch.randn(s, s, device="cuda", dtype=torch.bfloat16)
    us = timeit(lambda: a @ b.t(), reps=10)
    print(f"cuBLAS {s}^3 {us:.1f} us {2*s**3/us/1e6:.1f} TFLOP/s")
PY
