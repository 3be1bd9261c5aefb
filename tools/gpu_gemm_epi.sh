# FFN1 / FFN2 / QKV shapes at T = 5376 with every epilogue: mainloop-only (EPI_NONE = 7) vs stores vs fused epilogues
for shp in "5376 3072 768" "5376 768 3072" "5376 2304 768" "5376 768 768"; do
  for e in 7 0 1 2 3 5 6; do python tools/one_gemm.py 1 $e $shp 0 0 20 2>&1 | grep TFLOP; done
done
python - <<'PY'
import torch
from tools.bench_gemm import timeit
for (M, N, K) in ((5376, 3072, 768), (5376, 768, 3072), (5376, 2304, 768), (5376, 768, 768)):
    a = torch.randn(M, K, device="cuda", dtype=torch.bfloat16); b = torch.randn(N, K, device="cuda", dtype=torch.bfloat16)
    us = timeit(lambda: a @ b.t(), reps=20)
    print(f"cuBLAS {M}x{N}x{K} {us:.1f} us {2*M*N*K/us/1e6:.1f} TFLOP/s")
PY
