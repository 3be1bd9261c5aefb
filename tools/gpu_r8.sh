mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_gpu.log
summ() { tail -1 $1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value'],1), round(d['ms_per_step'],3), 'frac', round(d['roofline']['frac'],3), 'share', round(d['roofline']['share_of_step'],3), 'rr', d.get('recompute_ratio'), d['clocks']['sm_mhz'])" 2>&1 | tail -1; }
timeout 300 python bench.py --no-cpu-baseline --no-baselines > gpurun_out/bench_c.log 2>&1; echo "bench: $(summ gpurun_out/bench_c.log)"
for T in 2048 5120 8192; do timeout 300 python tools/bench_gemm.py $T "" 0,1 2>&1 | grep -v cuBLAS; done > gpurun_out/gemm_modes01.log; cat gpurun_out/gemm_modes01.log
