# In-step GEMM shape table (MIMOSE_PROBE_DUMP), a no-dropout A/B bound, and the ncu launch list at HEAD.
mkdir -p gpurun_out/explore
O=gpurun_out/explore
rm -f $O/probe.csv
MIMOSE_PROBE_DUMP=$O/probe.csv timeout 900 python bench.py --steps 60 --no-cpu-baseline --no-baselines > $O/bench.log 2>&1; echo "bench rc=$?"
tail -1 $O/bench.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('base', round(d['value'],1), round(d['ms_per_step'],3), 'frac', round(d['roofline']['frac'],3), d['clocks']['sm_mhz'])"
python tools/probe_summary.py $O/probe.csv > $O/probe_summary.txt; head -40 $O/probe_summary.txt
timeout 900 python bench.py --steps 60 --no-cpu-baseline --no-baselines --p-drop 0 > $O/bench_p0.log 2>&1; echo "bench p0 rc=$?"
tail -1 $O/bench_p0.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('p0', round(d['value'],1), round(d['ms_per_step'],3))"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches.csv \
  python bench.py --steps 2 --warmup 3 --no-baselines --no-cpu-baseline > /dev/null 2>&1; echo "ncu launches rc=$?"
python profiles/summarize_launches.py $O/launches.csv 40 > $O/launches_summary.txt; cat $O/launches_summary.txt
