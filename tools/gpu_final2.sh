mkdir -p gpurun_out
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?"; tail -2 gpurun_out/smoke.log
timeout 900 python bench.py > gpurun_out/bench_final.log 2>&1; echo "bench rc=$?"
tail -1 gpurun_out/bench_final.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value'],1), round(d['ms_per_step'],3), 'frac', round(d['roofline']['frac'],3), 'e2e', round(d['e2e']['value'],1), 'rr', d.get('recompute_ratio'), 'static', d.get('static_plan',{}).get('value'), 'sub', d.get('sublayer_units',{}).get('value'), 'cpu', d.get('cpu_baseline',{}).get('value'), d['clocks'])"
for c in bert-large roberta-large gpt2-medium; do
timeout 1200 python bench.py --config $c --steps 30 --no-cpu-baseline > gpurun_out/bench_final_$c.log 2>&1; echo "$c rc=$?"
tail -1 gpurun_out/bench_final_$c.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value'],1), round(d['ms_per_step'],3), 'frac', round(d['roofline']['frac'],3), 'rr', d.get('recompute_ratio'), 'static', d.get('static_plan',{}).get('value'), 'sub', d.get('sublayer_units',{}).get('value'), 'viol', d['mimose']['violations'])"
done
