"""One small training step through the C ABI, for compute-sanitizer runs
(tools/gpu_sanitize.sh): the fp32 toy (SIMT kernels) and a reduced bf16 BERT
(tcgen05 GEMMs and attention), each with a dropped (recomputed) layer, then
AdamW.  No oracle: the sanitizer checks memory accesses, races and barriers."""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_liaolysshfyctzlq23_b200 import binding as mb  # noqa: E402
from paper_conf_ipps_liaolysshfyctzlq23_b200 import workload as wl  # noqa: E402


def run(cfg, longest, budget_bytes):
    slab = torch.empty(budget_bytes, dtype=torch.uint8, device="cuda")
    ctx = mb.Mimose(cfg, budget_bytes, slab=slab, stream=torch.cuda.current_stream())
    ctx.set_params(wl.pack_params(cfg, wl.init_params(cfg, parity=True, seed=1)))
    b = wl.make_batch(cfg, longest, seed=2)
    p = mb.Plan()
    p.drop_mask = 1
    loss = ctx.forward(ctx.host_batch(b), p)
    ctx.backward()
    ctx.step(1e-4)
    torch.cuda.synchronize()
    ctx.close()
    return loss


if __name__ == "__main__":
    which = sys.argv[1] if len(sys.argv) > 1 else "both"
    if which in ("toy", "both"):
        print("toy fp32 loss", run(wl.CONFIGS["toy"], 23, 64 << 20))
    if which in ("bf16", "both"):
        cfg = wl.small_config("bert-base", n_layers=2, hidden=128, heads=2, ffn=256, vocab=500, max_pos=64,
                              n_seqs=8, seq_lo=8, seq_hi=40, pad=8)
        print("bf16 tcgen05 loss", run(cfg, 37, 256 << 20))
