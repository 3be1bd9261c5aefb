mkdir -p gpurun_out
timeout 300 python tools/bench_gemm.py 5120 "" 1,2,21,22 > gpurun_out/gemm_5120.log 2>&1
timeout 300 python tools/bench_gemm.py 2048 "" 1 > gpurun_out/gemm_2048.log 2>&1
timeout 300 python tools/bench_gemm.py 8192 "" 1 > gpurun_out/gemm_8192.log 2>&1
timeout 300 python tools/bench_gemm_modes.py 5120 > gpurun_out/gemm_modes.log 2>&1
timeout 300 ncu --set full --clock-control none --import-source on -k regex:k_gemm_tcp -s 3 -c 1 -o gpurun_out/wgr_ffn1 python tools/bench_gemm.py 5120 "wgr FFN1" 1 > gpurun_out/ncu_w.log 2>&1
timeout 300 ncu --set full --clock-control none --import-source on -k regex:k_gemm_tcp -s 3 -c 1 -o gpurun_out/fwd_ffn1 python tools/bench_gemm.py 5120 "fwd FFN1" 1 > gpurun_out/ncu_f.log 2>&1
for f in wgr_ffn1 fwd_ffn1; do ncu -i gpurun_out/$f.ncu-rep --page raw --csv > gpurun_out/${f}_raw.csv 2>/dev/null; done
