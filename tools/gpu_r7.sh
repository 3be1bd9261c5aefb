mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu.log
summ() { tail -1 $1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value'],1), round(d['ms_per_step'],3), 'frac', round(d['roofline']['frac'],3), 'share', round(d['roofline']['share_of_step'],3), 'rr', d.get('recompute_ratio'), d['clocks']['sm_mhz'])" 2>&1 | tail -1; }
timeout 300 python bench.py --no-cpu-baseline --no-baselines > gpurun_out/bench_b.log 2>&1; echo "bench: $(summ gpurun_out/bench_b.log)"
timeout 300 python tools/bench_gemm.py 5120 "gelu" 1 > gpurun_out/gemm_gelu.log 2>&1; cat gpurun_out/gemm_gelu.log
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 20000 --csv --log-file gpurun_out/launches.csv python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-baselines > gpurun_out/ncu_bench.log 2>&1; echo "ncu rc=$?"
