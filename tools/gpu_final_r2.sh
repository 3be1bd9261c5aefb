# Round-2 closing evidence at HEAD: GPU suite + smoke, every bench line, the ncu launch list and GEMM DRAM
# traffic of the default bench, the in-step CUPTI trace, and ncu --set full of the top kernels inside the bench.
mkdir -p gpurun_out/final
F=gpurun_out/final
timeout 2400 python -m pytest tests -m gpu -q -x > $F/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 $F/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $F/smoke.log 2>&1; echo "smoke rc=$?"; tail -3 $F/smoke.log
timeout 1500 python bench.py > $F/bench_bert-base.json 2> $F/bench_bert-base.err; echo "bb rc=$?"
for c in bert-large roberta-large gpt2-medium hetero t5-base; do
  timeout 900 python bench.py --config $c --steps 50 --no-cpu-baseline > $F/bench_$c.json 2> $F/bench_$c.err; echo "$c rc=$?"
done
python - <<'PY'
import json, glob
for f in sorted(glob.glob("gpurun_out/final/bench_*.json")):
    try:
        d = json.loads(open(f).read().strip().splitlines()[-1])
    except Exception as e:
        print(f, "ERR", e); continue
    print(d["config"]["workload"], round(d["value"], 1), "e2e", round(d["e2e"]["value"], 1), "ms", round(d["ms_per_step"], 3),
          "frac", round(d["roofline"]["frac"], 3), "rr", round(d.get("recompute_ratio", 0), 3),
          "static", round(d.get("static_plan", {}).get("value", 0), 1), "noc", round(d.get("no_ckpt", {}).get("value", 0), 1),
          "viol", d["mimose"]["violations"], "clk", d["clocks"]["sm_mhz"])
PY
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $F/launches.csv \
  python bench.py --steps 2 --warmup 3 --no-baselines --no-cpu-baseline > /dev/null 2>&1; echo "ncu launches rc=$?"
python profiles/summarize_launches.py $F/launches.csv 40 > $F/launches_summary.txt; head -25 $F/launches_summary.txt
timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum -k regex:k_gemm_tc --csv \
  --log-file $F/gemm_dram.csv python bench.py --steps 3 --warmup 3 --no-baselines --no-cpu-baseline > /dev/null 2>&1; echo "ncu dram rc=$?"
python tools/gemm_traffic.py $F/gemm_dram.csv $F/gemm_traffic.json; cat $F/gemm_traffic.json | head -5
timeout 600 python tools/trace_step.py bert-base 10 $F/trace_bb.json > $F/trace_bb.txt 2>&1; echo "trace rc=$?"; gzip -f $F/trace_bb.json
for k in "k_gemm_tcp:400:6" "k_attn_fwd_tc:20:1" "k_attn_bwd_tc:20:1" "k_ln_bwd:20:1" "k_ln_fwd:40:1" "k_adamw:10:1"; do
  IFS=: read name skip cnt <<< "$k"
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:$name -s $skip -c $cnt \
    -o $F/ncu_$name python bench.py --steps 2 --warmup 3 --no-baselines --no-cpu-baseline > /dev/null 2>&1; echo "ncu $name rc=$?"
done
ls -la $F
