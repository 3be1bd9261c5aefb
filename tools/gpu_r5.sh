mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu.log
summ() { tail -1 $1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value'],1), round(d['ms_per_step'],3), 'frac', round(d['roofline']['frac'],3), 'share', round(d['roofline']['share_of_step'],3), 'rr', d.get('recompute_ratio'), d['clocks']['sm_mhz'])" 2>&1 | tail -1; }
timeout 300 python bench.py --no-cpu-baseline --no-baselines > gpurun_out/bench_a.log 2>&1; echo "bench: $(summ gpurun_out/bench_a.log)"
timeout 300 python tools/bench_gemm.py 5120 "wgr" 1 > gpurun_out/gemm_wgr.log 2>&1; cat gpurun_out/gemm_wgr.log
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 20000 --csv --log-file gpurun_out/launches.csv python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-baselines > gpurun_out/ncu_bench.log 2>&1; echo "ncu rc=$?"
timeout 300 ncu --set full --clock-control none --import-source on -k regex:k_attn_fwd_tc -s 40 -c 1 -o gpurun_out/attn_fwd python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-baselines > gpurun_out/ncu_af.log 2>&1
timeout 300 ncu --set full --clock-control none --import-source on -k regex:k_attn_bwd_tc -s 20 -c 1 -o gpurun_out/attn_bwd python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-baselines > gpurun_out/ncu_ab.log 2>&1
timeout 300 ncu --set full --clock-control none --import-source on -k regex:k_gemm_tcp -s 3 -c 1 -o gpurun_out/fwd_ffn2 python tools/bench_gemm.py 5120 "fwd FFN2" 1 > gpurun_out/ncu_f2.log 2>&1
for f in attn_fwd attn_bwd fwd_ffn2; do ncu -i gpurun_out/$f.ncu-rep --page raw --csv > gpurun_out/${f}_raw.csv 2>/dev/null; done
