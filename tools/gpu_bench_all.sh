# Round-2 bench lines: BERT-base default (all arms + CPU oracle baseline), then every other config
mkdir -p gpurun_out/r2
timeout 1500 python bench.py > gpurun_out/r2/bench_bert-base.json 2> gpurun_out/r2/bench_bert-base.err; echo "bb rc=$?"
for c in bert-large roberta-large gpt2-medium hetero t5-base; do
  timeout 900 python bench.py --config $c --steps 50 --no-cpu-baseline > gpurun_out/r2/bench_$c.json 2> gpurun_out/r2/bench_$c.err; echo "$c rc=$?"
done
python - <<'PY'
import json, glob
for f in sorted(glob.glob("gpurun_out/r2/bench_*.json")):
    try:
        d = json.loads(open(f).read().strip().splitlines()[-1])
    except Exception as e:
        print(f, "ERR", e); continue
    print(d["config"]["workload"], round(d["value"], 1), "e2e", round(d["e2e"]["value"], 1), "ms", round(d["ms_per_step"], 3),
          "frac", round(d["roofline"]["frac"], 3), "rr", round(d.get("recompute_ratio", 0), 3),
          "static", round(d.get("static_plan", {}).get("value", 0), 1), "noc", round(d.get("no_ckpt", {}).get("value", 0), 1),
          "viol", d["mimose"]["violations"], "clk", d["clocks"]["sm_mhz"])
PY
