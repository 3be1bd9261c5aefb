# Round-2 evidence: sanitizer runs, host-issue timing, ncu launch list of the default bench, ncu --set full of
# the top GEMM and the attention kernels inside the bench
mkdir -p gpurun_out/r2prof
bash tools/gpu_sanitize.sh > gpurun_out/r2prof/sanitize_summary.txt 2>&1; cat gpurun_out/r2prof/sanitize_summary.txt
timeout 300 python tools/host_issue_time.py > gpurun_out/r2prof/host_issue.txt 2>&1; cat gpurun_out/r2prof/host_issue.txt
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r2prof/launches_r2.csv \
  python bench.py --steps 2 --warmup 3 --no-baselines --no-cpu-baseline > /dev/null 2>&1; echo "ncu launches rc=$?"
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:k_gemm_tcp -s 400 -c 6 \
  -o gpurun_out/r2prof/ncu_gemm_r2 python bench.py --steps 2 --warmup 3 --no-baselines --no-cpu-baseline > /dev/null 2>&1; echo "ncu gemm rc=$?"
timeout 900 ncu --set full --clock-control none -k regex:k_attn_bwd_tc -s 20 -c 1 \
  -o gpurun_out/r2prof/ncu_attn_bwd_r2 python bench.py --steps 2 --warmup 3 --no-baselines --no-cpu-baseline > /dev/null 2>&1; echo "ncu attn rc=$?"
timeout 900 ncu --set full --clock-control none -k regex:k_ln_bwd -s 20 -c 1 \
  -o gpurun_out/r2prof/ncu_ln_bwd_r2 python bench.py --steps 2 --warmup 3 --no-baselines --no-cpu-baseline > /dev/null 2>&1; echo "ncu ln rc=$?"
ls -la gpurun_out/r2prof
