mkdir -p gpurun_out
for T in 2048 5120 8192; do
timeout 300 python tools/bench_gemm.py $T "" 1,2,21,22 > gpurun_out/gemm_modes_$T.log 2>&1; echo "T=$T rc=$?"
done
