mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k units > gpurun_out/pytest_units.log 2>&1; echo "units rc=$?"; tail -4 gpurun_out/pytest_units.log
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu.log
timeout 1200 python bench.py --config gpt2-medium --steps 30 --no-cpu-baseline > gpurun_out/bench_g2u.log 2>&1; echo "g2 rc=$?"
tail -1 gpurun_out/bench_g2u.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value'],1), 'rr', d.get('recompute_ratio'), 'static', d.get('static_plan',{}).get('value'), 'sub', d.get('sublayer_units'))"
