# One default bench line (BERT-base, all arms) + BERT-large headline; JSON lines into gpurun_out/
mkdir -p gpurun_out
timeout 1500 python bench.py > gpurun_out/bench_bb.json 2> gpurun_out/bench_bb.err; echo "bb rc=$?"; tail -2 gpurun_out/bench_bb.err
python - <<'PY'
import json
d = json.loads(open("gpurun_out/bench_bb.json").read().strip().splitlines()[-1])
print("value", round(d["value"], 1), "e2e", round(d["e2e"]["value"], 1), "ms", round(d["ms_per_step"], 3),
      "frac", round(d["roofline"]["frac"], 3), "clk", d["clocks"]["sm_mhz"], "host_ms", d.get("host_issue_ms_per_step"))
for k in ("static_plan", "no_ckpt", "all_ckpt", "sublayer_units", "knapsack_units", "literal_budget", "normal_schedule"):
    print(k, {a: (round(b, 3) if isinstance(b, float) else b) for a, b in d.get(k, {}).items()})
print("recompute", d.get("recompute_ratio"), "incl_sheltered", d["incl_sheltered"]["value"], "tokens", d["tokens"])
PY
