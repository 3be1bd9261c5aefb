# A/B of the side-stream reductions (MIMOSE_AUX) on the default BERT-base bench, two runs each
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -q -x -k "not fullsize" > gpurun_out/pytest_aux.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_aux.log
for v in 1 0 1 0; do
  MIMOSE_AUX=$v timeout 600 python bench.py --no-baselines --no-cpu-baseline > gpurun_out/ab_aux_$v.json 2>/dev/null
  python -c "import json; d=json.loads(open('gpurun_out/ab_aux_$v.json').read().strip().splitlines()[-1]); print('AUX=$v', round(d['value'],1), round(d['ms_per_step'],3), d['clocks']['sm_mhz'])"
done
