"""In-step kernel timeline of the bench workload through CUPTI (torch.profiler):
every kernel the library launches on every stream, with device timestamps, over
a few warm steps -- unlike an ncu launch list (cold cache, serialised), this is
what the step really spends, with the side-stream overlap.

    python tools/trace_step.py [config] [steps] [out.json]

Prints, per kernel on the compute stream, its critical-path increment (how far
it pushes the stream's busy frontier: durations overlap under programmatic
dependent launch, so raw durations are not additive) and the idle gaps before
it (waits on side-stream events), then per-kernel totals on the side streams."""
import collections
import json
import os
import re
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_liaolysshfyctzlq23_b200 import binding as mb  # noqa: E402
from paper_conf_ipps_liaolysshfyctzlq23_b200 import workload as wl  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "bert-base"
steps = int(sys.argv[2]) if len(sys.argv) > 2 else 10
out = sys.argv[3] if len(sys.argv) > 3 else None
cfg = wl.CONFIGS[name]
stream = torch.cuda.current_stream()
pc = mb.Mimose(cfg, 0)
C0 = pc.stats()["persistent_bytes"]
P0 = pc.dry_run(cfg.n_seqs, cfg.max_seq, [])
LB = pc.dry_run(cfg.n_seqs, cfg.max_seq, range(cfg.n_layers))
M = max(C0 + int(cfg.budget_frac * (P0 - C0)), LB)
pc.close()
slab = torch.empty(M, dtype=torch.uint8, device="cuda")
ctx = mb.Mimose(cfg, M, slab=slab, stream=stream, enforce_budget=1, use_tc=1)
ctx.set_params(wl.pack_params(cfg, wl.init_params(cfg)))
ctx.set_optimizer(1e-5, fused=True)
sched = wl.length_schedule(cfg, 10 + 5 + steps)
n = 0
while ctx.phase == mb.PHASE_SHELTERED:
    b = wl.make_batch(cfg, sched[n % 10], seed=wl.batch_seed(cfg, 10**6 + n, 0))
    ctx.collect(ctx.host_batch(b), want_loss=False)
    ctx.backward()
    ctx.step(1e-5)
    n += 1
batches = [wl.make_batch(cfg, sched[10 + i], seed=wl.batch_seed(cfg, 10 + i, 0)) for i in range(5 + steps)]
dev = [[torch.tensor(np.ascontiguousarray(x, np.int32)).cuda() for x in (b.input_ids, b.token_type, b.lengths, b.labels)]
       for b in batches]


def one(i):
    b = batches[i]
    bs = mb.Mimose.batch_struct(*dev[i], b.n_seqs, b.seq_len, False)
    ctx.forward(bs, ctx.plan(b.input_size), want_loss=False)
    ctx.backward()
    ctx.step(1e-5)


for i in range(5):
    one(i)
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
with torch.profiler.profile(activities=[torch.profiler.ProfilerActivity.CUDA]) as prof:
    e0.record(stream)
    for i in range(5, 5 + steps):
        one(i)
    e1.record(stream)
    torch.cuda.synchronize()
step_ms = e0.elapsed_time(e1) / steps
path = out or "/tmp/trace_step.json"
prof.export_chrome_trace(path)
ev = [e for e in json.load(open(path))["traceEvents"] if e.get("cat") == "kernel"]
by_stream = collections.defaultdict(list)
for e in ev:
    by_stream[e["args"]["stream"]].append(e)
main = max(by_stream, key=lambda s: len(by_stream[s]))   # the compute stream issues most launches
t0 = min(e["ts"] for e in ev)
t1 = max(e["ts"] + e["dur"] for e in ev)


def union(es):
    iv = sorted((e["ts"], e["ts"] + e["dur"]) for e in es)
    tot, cs, ce = 0.0, None, None
    for s, f in iv:
        if ce is None or s > ce:
            if ce is not None:
                tot += ce - cs
            cs, ce = s, f
        else:
            ce = max(ce, f)
    return tot + (ce - cs if ce is not None else 0.0)


span = t1 - t0
print(f"# {name}: {steps} steps, {step_ms:.3f} ms/step (events), trace span {span / 1000 / steps:.3f} ms/step")
for s, es in sorted(by_stream.items(), key=lambda x: -len(x[1])):
    print(f"# stream {s}{' (compute)' if s == main else ''}: {len(es) / steps:.0f} kernels/step, "
          f"busy {union(es) / span:.3f} of the span")
print(f"# all streams: busy {union(ev) / span:.3f} of the span")
def nm(e):   # the kernel name without its argument list (names may start with "(anonymous namespace)::")
    n = e["name"].replace("(anonymous namespace)::", "").replace("void ", "").replace("mimose::", "")
    return re.sub(r"\(.*", "", n)[:60]



inc, gap = collections.defaultdict(lambda: [0, 0.0]), collections.defaultdict(lambda: [0, 0.0])
m = sorted(by_stream[main], key=lambda e: e["ts"])
front = m[0]["ts"]
for e in m:
    s0, f0 = e["ts"], e["ts"] + e["dur"]
    if s0 > front:
        gap[nm(e)][0] += 1
        gap[nm(e)][1] += s0 - front
    inc[nm(e)][0] += 1
    inc[nm(e)][1] += max(0.0, f0 - max(s0, front))
    front = max(front, f0)
print(f"\n## compute stream critical path: {sum(v[1] for v in inc.values()) / 1000 / steps:.3f} ms/step of kernels, "
      f"{sum(v[1] for v in gap.values()) / 1000 / steps:.3f} ms/step idle")
print(f"{'share_step':>10} {'us/step':>9} {'n/step':>7} {'avg_us':>8}  kernel (increment)")
for k, (c, d) in sorted(inc.items(), key=lambda x: -x[1][1])[:25]:
    print(f"{100 * d / 1000 / steps / step_ms:9.1f}% {d / steps:9.1f} {c / steps:7.1f} {d / c:8.2f}  {k}")
print(f"{'share_step':>10} {'us/step':>9} {'n/step':>7} {'avg_us':>8}  idle gap before")
for k, (c, d) in sorted(gap.items(), key=lambda x: -x[1][1])[:8]:
    print(f"{100 * d / 1000 / steps / step_ms:9.1f}% {d / steps:9.1f} {c / steps:7.1f} {d / c:8.2f}  {k}")
for s in [x for x in by_stream if x != main]:
    agg = collections.defaultdict(lambda: [0, 0.0])
    for e in by_stream[s]:
        agg[nm(e)][0] += 1
        agg[nm(e)][1] += e["dur"]
    tot = sum(v[1] for v in agg.values())
    print(f"\n## stream {s}: {tot / 1000 / steps:.3f} ms/step of kernel durations")
    print(f"{'share_step':>10} {'us/step':>9} {'n/step':>7} {'avg_us':>8}  kernel")
    for k, (c, d) in sorted(agg.items(), key=lambda x: -x[1][1])[:12]:
        print(f"{100 * d / 1000 / steps / step_ms:9.1f}% {d / steps:9.1f} {c / steps:7.1f} {d / c:8.2f}  {k}")
