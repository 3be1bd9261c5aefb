# GPU suite (no full-size) + encoder-decoder + the default bench line
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -x -k "not fullsize" > gpurun_out/pytest_q.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_q.log
timeout 600 python bench.py --no-baselines --no-cpu-baseline > gpurun_out/bench_q.json 2>/dev/null
python -c "import json; d=json.loads(open('gpurun_out/bench_q.json').read().strip().splitlines()[-1]); print('BB', round(d['value'],1), round(d['ms_per_step'],3), d['clocks']['sm_mhz'])"
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -3
