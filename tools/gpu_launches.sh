# ncu launch list of the default bench command (cold-cache, serialised per-launch times)
mkdir -p gpurun_out/launches
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches/launches.csv \
  python bench.py --steps 2 --warmup 3 --no-baselines --no-cpu-baseline > /dev/null 2>&1; echo "ncu launches rc=$?"
python profiles/summarize_launches.py gpurun_out/launches/launches.csv 40 > gpurun_out/launches/summary.txt; cat gpurun_out/launches/summary.txt
