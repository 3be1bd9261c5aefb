# Same-box A/B of two builds of libmimose.so (ab_so/libmimose_base.so vs ab_so/libmimose_new.so):
# GPU tests on the new build, then alternating BERT-base bench runs.
#   bash tools/gpu_ab_so.sh [pytest files...]
mkdir -p gpurun_out/ab
LIB=paper_conf_ipps_liaolysshfyctzlq23_b200/libmimose.so
cp ab_so/libmimose_new.so $LIB
if [ $# -gt 0 ]; then
  timeout 1500 python -m pytest "$@" -x -q -m gpu > gpurun_out/ab/pytest.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/ab/pytest.log
fi
for i in 1 2 3; do
  for v in base new; do
    cp ab_so/libmimose_$v.so $LIB
    timeout 600 python bench.py --steps 60 --no-cpu-baseline --no-baselines ${BENCH_ARGS} > gpurun_out/ab/b_$v.log 2>&1
    tail -1 gpurun_out/ab/b_$v.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$v', round(d['value'],1), round(d['ms_per_step'],3), d['clocks']['sm_mhz'])"
  done
done
cp ab_so/libmimose_new.so $LIB
