mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu.log
timeout 300 python tools/bench_gemm.py 5120 "drop" 1 > gpurun_out/gdrop.log 2>&1; grep "mode=1" gpurun_out/gdrop.log
timeout 900 python bench.py --no-cpu-baseline > gpurun_out/bench.log 2>&1; echo "bench rc=$?"
tail -1 gpurun_out/bench.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value'],1), round(d['ms_per_step'],3), 'frac', round(d['roofline']['frac'],3), 'share', round(d['roofline']['share_of_step'],3), 'rr', d.get('recompute_ratio'), 'sub', d.get('sublayer_units',{}).get('value'), d['clocks']['sm_mhz'])"
