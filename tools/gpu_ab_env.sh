# Same-box A/B of one build under two environments: GPU tests first (optional), then alternating BERT-base runs.
#   A="MIMOSE_X=0" B="MIMOSE_X=1" bash tools/gpu_ab_env.sh [pytest files...]
mkdir -p gpurun_out/ab
if [ $# -gt 0 ]; then
  timeout 1500 python -m pytest "$@" -x -q -m gpu > gpurun_out/ab/pytest.log 2>&1; echo "pytest rc=$?"; tail -5 gpurun_out/ab/pytest.log
fi
for i in 1 2 3; do
  for v in "$A" "$B"; do
    env $v timeout 600 python bench.py --steps 60 --no-cpu-baseline --no-baselines ${BENCH_ARGS} > gpurun_out/ab/b.log 2>&1
    tail -1 gpurun_out/ab/b.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$v', round(d['value'],1), round(d['ms_per_step'],3), d['clocks']['sm_mhz'])" || tail -5 gpurun_out/ab/b.log
  done
done
