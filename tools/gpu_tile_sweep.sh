# Tile width per step GEMM shape: modes 12 (128x256), 13 (128x128), 17 (CTA pair 256x256), 1 (default) at three token counts.
mkdir -p gpurun_out/sweep
for T in 2560 5376 8192; do
  timeout 600 python tools/bench_gemm.py $T "" 12,13,17,1 > gpurun_out/sweep/T$T.txt 2>&1; echo "T=$T rc=$?"
done
grep -v cuBLAS gpurun_out/sweep/T*.txt
