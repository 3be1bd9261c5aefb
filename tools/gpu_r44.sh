mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?"; tail -3 gpurun_out/smoke.log
timeout 900 python bench.py --no-cpu-baseline --no-baselines > gpurun_out/bench.log 2>&1; echo "bench rc=$?"
tail -1 gpurun_out/bench.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value'],1), round(d['ms_per_step'],3), 'frac', round(d['roofline']['frac'],3), 'traffic', d['roofline']['traffic'], d['clocks']['sm_mhz'])"
for k in "256, \(int\)2," "256, \(int\)3," "256, \(int\)6, \(bool\)0, \(bool\)1"; do
  tag=$(echo "$k" | tr -cd '0-9')
  timeout 600 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k "regex:k_gemm_tcp<\(int\)$k" -s 20 -c 1 -o gpurun_out/full_gemm_$tag python bench.py --steps 2 --warmup 3 --no-baselines --no-cpu-baseline > gpurun_out/ncu_full_gemm_$tag.log 2>&1; echo "$tag rc=$?"
done
ls gpurun_out/*.ncu-rep
