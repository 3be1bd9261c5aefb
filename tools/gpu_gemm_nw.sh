# epilogue stores A/B: mode 1 (staged through smem) vs mode 16 (direct) on the step shapes
for shp in "5376 3072 768" "5376 768 3072" "5376 2304 768" "5376 768 768"; do
  for e in 0 2 3 4 5 6; do for m in 1 16; do python tools/one_gemm.py $m $e $shp 0 0 20 2>&1 | grep TFLOP; done; done
done
