mkdir -p gpurun_out
timeout 120 python tools/bench_gemm.py 5120 "" 1 > gpurun_out/gemm_m1.log 2>&1
timeout 300 ncu --set full --clock-control none --import-source on -k regex:k_gemm_tcp -s 3 -c 1 -o gpurun_out/gelu_fwd python tools/bench_gemm.py 5120 "FFN1 gelu" 1 > gpurun_out/ncu_gf.log 2>&1
timeout 300 ncu --set full --clock-control none --import-source on -k regex:k_gemm_tcp -s 3 -c 1 -o gpurun_out/gelu_bwd python tools/bench_gemm.py 5120 "FFN2 gelu'" 1 > gpurun_out/ncu_gb.log 2>&1
timeout 300 ncu --set full --clock-control none --import-source on -k regex:k_gemm_tcp -s 3 -c 1 -o gpurun_out/bias_qkv python tools/bench_gemm.py 5120 "QKV  bias" 1 > gpurun_out/ncu_bq.log 2>&1
timeout 300 python bench.py --steps 20 --warmup 5 --no-cpu-baseline --no-baselines > gpurun_out/bench.log 2>&1
tail -1 gpurun_out/bench.log
