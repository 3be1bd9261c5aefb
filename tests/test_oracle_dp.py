"""c-J data-parallel semantics on the oracle with a real 2-rank gloo group (CPU).

Gradient of a DP step = mean over ranks of per-rank mean-loss gradients; with
equal per-rank batches (shared S_t, DESIGN "Multi-GPU") this equals the
gradient of the mean loss over the concatenated global batch.  Dropout off
(p=0): masks are per-rank by design (site word carries the rank)."""
import os
import socket

import numpy as np
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from oracle import model as om
from paper_conf_ipps_liaolysshfyctzlq23_b200 import workload as wl


def cfg_():
    return wl.small_config("toy", n_layers=2, hidden=16, heads=2, ffn=32, vocab=40,
                           max_pos=16, first_tok=3, cls_id=1, sep_id=2, pad_id=0,
                           n_seqs=4, head=wl.HEAD_MC, n_choices=2)


def shard(cfg, rank, S=6):
    return wl.make_batch(cfg, S, seed=100 + rank)


def _worker(rank, world, port, out):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    cfg = cfg_()
    params = wl.init_params(cfg, parity=True, seed=2)
    _, G = om.train_step_grads(cfg, params, shard(cfg, rank), 5, 0, rank=rank, p=0.0)
    flat = torch.tensor(np.concatenate([G[n].ravel() for n, _ in wl.param_spec(cfg)]))
    dist.all_reduce(flat)
    flat /= world
    if rank == 0:
        out.put(flat.numpy())
    dist.barrier()
    dist.destroy_process_group()


def free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def test_dp_mean_equals_concatenated_batch():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    got = q.get(timeout=120)
    for p in procs:
        p.join(60)
        assert p.exitcode == 0
    cfg = cfg_()
    params = wl.init_params(cfg, parity=True, seed=2)
    b0, b1 = shard(cfg, 0), shard(cfg, 1)
    cat = wl.Batch(np.concatenate([b0.input_ids, b1.input_ids]),
                   np.concatenate([b0.token_type, b1.token_type]),
                   np.concatenate([b0.lengths, b1.lengths]),
                   np.concatenate([b0.labels, b1.labels]), b0.seq_len)
    cfg2 = wl.small_config("toy", **{**cfg.__dict__, "n_seqs": 8})
    _, G = om.train_step_grads(cfg2, params, cat, 5, 0, p=0.0)
    ref = np.concatenate([G[n].ravel() for n, _ in wl.param_spec(cfg)])
    assert np.abs(got - ref).max() <= 1e-12 * max(1.0, np.abs(ref).max())


