mkdir -p gpurun_out
timeout 1500 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/kern_r1o.csv python bench.py --steps 2 --warmup 3 --no-baselines --no-cpu-baseline > gpurun_out/ncu_kern_o.log 2>&1; echo "metrics rc=$?"
python tools/kernel_roofline.py gpurun_out/kern_r1o.csv > gpurun_out/kernels_r1o_summary.txt; head -25 gpurun_out/kernels_r1o_summary.txt
python tools/gemm_traffic.py gpurun_out/kern_r1o.csv gpurun_out/gemm_traffic.json
for k in "k_gemm_tcp<256, 2, " "k_gemm_tcp<256, 3, " "k_gemm_tcp<256, 6, 0, 1>" "k_attn_fwd_tc"; do
  tag=$(echo "$k" | tr -cd 'a-z0-9_'); 
  timeout 600 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k "regex:$k" -s 20 -c 1 -o gpurun_out/full_$tag python bench.py --steps 2 --warmup 3 --no-baselines --no-cpu-baseline > gpurun_out/ncu_full_$tag.log 2>&1; echo "$tag rc=$?"
done
ls gpurun_out/*.ncu-rep
