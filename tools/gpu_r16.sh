mkdir -p gpurun_out
for m in 12 22; do python tools/one_gemm.py $m 7 8192 3072 768; done
timeout 300 ncu --set full --clock-control none --import-source on -k regex:k_gemm_tc -s 3 -c 1 -o gpurun_out/ncu_m12 python tools/one_gemm.py 12 7 8192 3072 768 0 0 5 > /dev/null 2>&1; echo "rc=$?"
timeout 300 ncu --set full --clock-control none --import-source on -k regex:k_gemm_tc -s 3 -c 1 -o gpurun_out/ncu_m22 python tools/one_gemm.py 22 7 8192 3072 768 0 0 5 > /dev/null 2>&1; echo "rc=$?"
