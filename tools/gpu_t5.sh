# tiled cross-attention round: full GPU suite, then the t5-base bench line (src 17-460)
mkdir -p gpurun_out/r2
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_all.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_all.log
timeout 900 python bench.py --config t5-base --steps 50 --no-cpu-baseline > gpurun_out/r2/bench_t5-base.json 2> gpurun_out/r2/bench_t5-base.err; echo "t5 rc=$?"
python - <<'PY'
import json
d = json.loads(open("gpurun_out/r2/bench_t5-base.json").read().strip().splitlines()[-1])
print(d["config"]["workload"], round(d["value"], 1), "e2e", round(d["e2e"]["value"], 1), "ms", round(d["ms_per_step"], 3),
      "frac", round(d["roofline"]["frac"], 3), "rr", round(d.get("recompute_ratio", 0), 3),
      "static", round(d.get("static_plan", {}).get("value", 0), 1), "noc", round(d.get("no_ckpt", {}).get("value", 0), 1),
      "knap", round(d.get("knapsack_layers", {}).get("value", 0), 1),
      "viol", d["mimose"]["violations"], "clk", d["clocks"]["sm_mhz"])
PY
