# TMA-store epilogue: correctness (GEMM tests incl. mode 16) and the A/B on the step shapes
timeout 900 python -m pytest tests/test_gpu_gemm.py -q -x 2>&1 | tail -3
for shp in "5376 3072 768" "5376 768 3072" "5376 2304 768" "5376 768 768"; do
  for e in 0 2 3 4 5 6; do for m in 1 16; do python tools/one_gemm.py $m $e $shp 0 0 20 2>&1 | grep TFLOP; done; done
done
