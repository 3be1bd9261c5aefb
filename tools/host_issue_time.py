"""Host time the library spends issuing one BERT-base step (plan + forward +
backward + step) with the launch queue empty, against the step's GPU time.
If the host issues a step much faster than the GPU runs it, the GPU never
waits for launches and CUDA-graph capture cannot raise throughput.

    python tools/host_issue_time.py        (on the GPU box)
"""
import os
import sys
import time

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_liaolysshfyctzlq23_b200 import binding as mb  # noqa: E402
from paper_conf_ipps_liaolysshfyctzlq23_b200 import workload as wl  # noqa: E402

cfg = wl.CONFIGS["bert-base"]
probe = mb.Mimose(cfg, 0)
C0 = probe.stats()["persistent_bytes"]
P0 = probe.dry_run(cfg.n_seqs, cfg.max_seq, [])
LB = probe.dry_run(cfg.n_seqs, cfg.max_seq, range(cfg.n_layers))
M = max(C0 + int(cfg.budget_frac * (P0 - C0)), LB)
slab = torch.empty(M, dtype=torch.uint8, device="cuda")
st = torch.cuda.current_stream()
ctx = mb.Mimose(cfg, M, slab=slab, stream=st)
ctx.set_params(wl.pack_params(cfg, wl.init_params(cfg)))
ctx.set_optimizer(1e-5, fused=True)
sched = wl.length_schedule(cfg, 80)
i = 0
while ctx.phase == mb.PHASE_SHELTERED:
    b = wl.make_batch(cfg, sched[i], seed=i)
    ctx.collect(ctx.host_batch(b), want_loss=False)
    ctx.backward()
    ctx.step(1e-5)
    i += 1
bs = [wl.make_batch(cfg, L, seed=100 + j) for j, L in enumerate(sched[i:i + 40])]
dev = [[torch.tensor(np.ascontiguousarray(x, np.int32)).cuda() for x in (b.input_ids, b.token_type, b.lengths, b.labels)]
       for b in bs]
structs = [mb.Mimose.batch_struct(*d, b.n_seqs, b.seq_len, False) for d, b in zip(dev, bs)]
for j in range(5):
    ctx.forward(structs[j], ctx.plan(bs[j].input_size), False)
    ctx.backward()
    ctx.step(1e-5)
host, gpu = [], []
for j in range(5, 40):
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(st)
    t0 = time.perf_counter()
    ctx.forward(structs[j], ctx.plan(bs[j].input_size), False)
    ctx.backward()
    ctx.step(1e-5)
    host.append(1000 * (time.perf_counter() - t0))
    e1.record(st)
    torch.cuda.synchronize()
    gpu.append(e0.elapsed_time(e1))
print(f"host issue {np.mean(host):.3f} ms / step, GPU {np.mean(gpu):.3f} ms / step (BERT-base, 35 steps, "
      f"launch queue empty before each step)")
