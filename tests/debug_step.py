"""Debug helper (not a test): one collect + one plan-driven step at a config's width."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from oracle import memsim as om
from paper_conf_ipps_liaolysshfyctzlq23_b200 import workload as wl, binding as mb
name = sys.argv[1] if len(sys.argv) > 1 else "bert-base"
L = int(sys.argv[2]) if len(sys.argv) > 2 else 2
cfg = wl.small_config(name, n_layers=L)
sz = om.sizes(cfg, cfg.n_seqs, cfg.max_seq)
M = om.no_ckpt_peak(sz)
slab = torch.empty(M, dtype=torch.uint8, device="cuda")
ctx = mb.Mimose(cfg, M, slab=slab, stream=torch.cuda.current_stream())
ctx.set_params(wl.pack_params(cfg, wl.init_params(cfg)))
print("params set", flush=True)
b = wl.make_batch(cfg, cfg.seq_hi, seed=1)
print("collect loss", ctx.collect(ctx.host_batch(b)), flush=True)
ctx.backward(); torch.cuda.synchronize(); print("bwd ok", flush=True)
ctx.step(1e-4); torch.cuda.synchronize(); print("step ok", flush=True)
p = mb.Plan(); p.drop_mask = 1
print("fwd loss", ctx.forward(ctx.host_batch(b), p), flush=True)
ctx.backward(); torch.cuda.synchronize(); print("ok", ctx.stats()["peak_bytes"], flush=True)
