# ncu --set full of one 8192^3 GEMM: the library kernel and cuBLAS
mkdir -p gpurun_out
ncu --set full --clock-control none -k regex:k_gemm_tcp -s 2 -c 1 -o gpurun_out/gemm8k_ours -f python tools/one_gemm.py 1 0 8192 8192 8192 0 0 3 > /dev/null 2>&1
ncu --set full --clock-control none -k regex:"gemm|Kernel|sm100" -s 2 -c 1 -o gpurun_out/gemm8k_cublas -f python - <<'PY' > /dev/null 2>&1
import torch
a = torch.randn(8192, 8192, device="cuda", dtype=torch.bfloat16); b = torch.randn(8192, 8192, device="cuda", dtype=torch.bfloat16)
for _ in range(4): c = a @ b.t()
torch.cuda.synchronize()
PY
ls -la gpurun_out/*.ncu-rep
