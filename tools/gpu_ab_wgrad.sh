# side-stream weight gradients: GPU tests + A/B on the default BERT-base bench (MIMOSE_AUX_WGRAD)
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -q -x -k "not fullsize" > gpurun_out/pytest_wg.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_wg.log
for v in 1 0 1 0; do
  MIMOSE_AUX_WGRAD=$v timeout 600 python bench.py --no-baselines --no-cpu-baseline > gpurun_out/ab_wg_$v.json 2>/dev/null
  python -c "import json; d=json.loads(open('gpurun_out/ab_wg_$v.json').read().strip().splitlines()[-1]); print('AUX_WGRAD=$v', round(d['value'],1), round(d['ms_per_step'],3), d['clocks']['sm_mhz'], 'frac', round(d['roofline']['frac'],3))"
done
