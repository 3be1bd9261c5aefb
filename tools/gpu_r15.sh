mkdir -p gpurun_out
MODES=12,14 timeout 300 python tools/bench_gemm_modes.py 5120 > gpurun_out/sk_none_5120.log 2>&1; cat gpurun_out/sk_none_5120.log
timeout 300 ncu --set full --clock-control none --import-source on -k regex:k_gemm_tcp -s 3 -c 1 -o gpurun_out/ncu_sk_gf python tools/bench_gemm.py 5120 "FFN1 gelu" 1 > gpurun_out/ncu_sk_gf.log 2>&1; echo "ncu rc=$?"
