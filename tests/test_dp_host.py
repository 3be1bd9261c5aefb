"""N > 1 host path on CPU with a real 2-rank gloo group: every rank runs its own
host-only library context on its own batches of the SHARED length schedule
(DESIGN "Multi-GPU"), and all ranks derive bit-identical plans without any plan
broadcast — equal to the oracle planner's."""
import os
import socket

import numpy as np
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from oracle import estimator as oe
from oracle import memsim as om
from oracle import planner as op
from paper_conf_ipps_liaolysshfyctzlq23_b200 import workload as wl


def _budget(cfg):
    sz = om.sizes(cfg, cfg.n_seqs, cfg.max_seq)
    return max(sz.C + int(cfg.budget_frac * (om.no_ckpt_peak(sz) - sz.C)), om.lower_bound(sz))


def _worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_ipps_liaolysshfyctzlq23_b200 import binding as mb
    cfg = wl.CONFIGS["bert-base"]
    ctx = mb.Mimose(cfg, _budget(cfg))                 # host-only: accounting, estimator, planner
    sched = wl.length_schedule(cfg, 80)                # shared S_t
    i = 0
    while ctx.phase == mb.PHASE_SHELTERED:
        b = wl.make_batch(cfg, sched[i], seed=wl.batch_seed(cfg, i, rank))   # per-rank data
        ctx.collect(ctx.host_batch(b), want_loss=False)
        ctx.backward()
        i += 1
    masks = []
    for L_t in sched[i:]:
        x = cfg.n_seqs * wl.roundup(L_t, cfg.pad)
        masks.append(ctx.plan(x).drop_mask)
    t = torch.tensor(masks, dtype=torch.int64)
    allm = [torch.zeros_like(t) for _ in range(world)]
    dist.all_gather(allm, t)
    if rank == 0:
        q.put((i, [m.tolist() for m in allm]))
    dist.barrier()
    dist.destroy_process_group()


def test_two_ranks_derive_identical_plans():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    n_sheltered, allm = q.get(timeout=300)
    for p in procs:
        p.join(60)
        assert p.exitcode == 0
    assert allm[0] == allm[1]
    # == the oracle pipeline on the same schedule
    cfg = wl.CONFIGS["bert-base"]
    sched = wl.length_schedule(cfg, 80)
    samples, seen = [], set()
    for L_t in sched[:n_sheltered]:
        S = wl.roundup(L_t, cfg.pad)
        if cfg.n_seqs * S not in seen:
            seen.add(cfg.n_seqs * S)
            c = om.collect_samples(om.sizes(cfg, cfg.n_seqs, S))
            c["x"] = cfg.n_seqs * S
            samples.append(c)
    est = oe.Estimator(samples)
    want = []
    for L_t in sched[n_sheltered:]:
        st, dropped, _ = op.plan(est.predict(cfg.n_seqs * wl.roundup(L_t, cfg.pad)), _budget(cfg))
        want.append(sum(1 << l for l in dropped))
    assert allm[0] == want
