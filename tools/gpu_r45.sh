mkdir -p gpurun_out/tmp
for k in "256, \(int\)2," "256, \(int\)3," "256, \(int\)6, \(bool\)0, \(bool\)1"; do
  tag=$(echo "$k" | tr -cd '0-9')
  timeout 600 ncu --set full --clock-control none --kernel-name-base demangled -k "regex:k_gemm_tcp<\(int\)$k" -s 20 -c 1 -o gpurun_out/tmp/full_gemm_$tag python bench.py --steps 2 --warmup 3 --no-baselines --no-cpu-baseline > /dev/null 2>&1; echo "$tag rc=$?"
  python tools/ncu_summary.py gpurun_out/tmp/full_gemm_$tag.ncu-rep > gpurun_out/ncu_full_gemm_${tag}_r1p.txt
done
rm -rf gpurun_out/tmp
cat gpurun_out/ncu_full_gemm_*_r1p.txt
