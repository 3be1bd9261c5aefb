# encoder-decoder GPU tests, the rest of the GPU suite, and the BERT-base bench line
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_encdec.py -q -x > gpurun_out/encdec.log 2>&1; echo "encdec rc=$?"; tail -4 gpurun_out/encdec.log
timeout 1500 python -m pytest tests -m gpu -q -x -k "not encdec" > gpurun_out/pytest_rest.log 2>&1; echo "rest rc=$?"; tail -3 gpurun_out/pytest_rest.log
timeout 600 python bench.py --no-baselines --no-cpu-baseline > gpurun_out/bench_quick.json 2>/dev/null
python -c "import json; d=json.loads(open('gpurun_out/bench_quick.json').read().strip().splitlines()[-1]); print('BB', round(d['value'],1), round(d['ms_per_step'],3), d['clocks']['sm_mhz'])"
