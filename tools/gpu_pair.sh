# CTA-pair GEMM: tests (timeout-guarded), then the A/B on step shapes and 8192^3
timeout 600 python -m pytest tests/test_gpu_gemm.py -q -x 2>&1 | tail -4
for shp in "5376 3072 768" "5376 768 3072" "5376 2304 768" "5376 768 768" "8192 8192 8192"; do
  for e in 7 0 2 3 5; do for m in 1 17; do timeout 60 python tools/one_gemm.py $m $e $shp 0 0 20 2>&1 | grep TFLOP; done; done
done
for m in 1 17; do timeout 60 python tools/one_gemm.py $m 6 768 3072 5376 1 1 20 2>&1 | grep TFLOP; done
