# After the tiled-attention change: GPU suite + smoke, and the bench lines of the configs that use it.
mkdir -p gpurun_out/final2
F=gpurun_out/final2
timeout 2400 python -m pytest tests -m gpu -q -x > $F/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 $F/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $F/smoke.log 2>&1; echo "smoke rc=$?"; tail -3 $F/smoke.log
for c in bert-large roberta-large gpt2-medium t5-base; do
  timeout 900 python bench.py --config $c --steps 50 --no-cpu-baseline > $F/bench_$c.json 2> $F/bench_$c.err; echo "$c rc=$?"
done
python - <<'PY'
import json, glob
for f in sorted(glob.glob("gpurun_out/final2/bench_*.json")):
    d = json.loads(open(f).read().strip().splitlines()[-1])
    print(d["config"]["workload"], round(d["value"], 1), "e2e", round(d["e2e"]["value"], 1), "rr", round(d.get("recompute_ratio", 0), 3),
          "static", round(d.get("static_plan", {}).get("value", 0), 1), "noc", round(d.get("no_ckpt", {}).get("value", 0), 1),
          "viol", d["mimose"]["violations"], "clk", d["clocks"]["sm_mhz"])
PY
