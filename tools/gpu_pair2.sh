# CTA-pair GEMM on the large-model shapes: H = 1024 layers at T = 8192, GPT-2 LM-head chunk GEMMs
for spec in "8192 4096 1024 0 0" "8192 1024 4096 0 0" "8192 3072 1024 0 0" "1024 4096 8192 1 1" "2048 1024 50264 0 1" "50264 1024 2048 1 1" "4096 1024 4096 0 0"; do
  for e in 0 6; do for m in 1 17; do timeout 60 python tools/one_gemm.py $m $e $spec 20 2>&1 | grep TFLOP; done; done
done
