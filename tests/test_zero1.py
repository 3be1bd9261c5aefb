"""ZeRO-1 optimizer-state sharding (parameters,
gradients and optimizer states are the input-independent part of the
footprint).  Host-side pins (no GPU): the library's persistent bytes and
arena peaks with ZeRO-1 at world 1/2/4/8 equal the oracle memory model, the
bucket padding splits every bucket into equal shards, the per-parameter
persistent cost falls from 18 B to 6 + 12/world B, and under the same budget
the planner drops no more layers than without sharding."""
import numpy as np
import pytest

from oracle import memsim as om
from oracle import planner as op
from paper_conf_ipps_liaolysshfyctzlq23_b200 import binding as mb
from paper_conf_ipps_liaolysshfyctzlq23_b200 import workload as wl

CFGS = ["toy", "bert-base", "bert-large", "roberta-large", "gpt2-medium"]


def a16(n):
    return (n + 15) // 16 * 16


@pytest.mark.parametrize("name", CFGS)
@pytest.mark.parametrize("world", [1, 2, 4, 8])
def test_zero1_persistent_bytes(name, world):
    cfg = wl.CONFIGS[name]
    npad = om.padded_numel(cfg, world, True)
    assert npad % (64 * world) == 0
    for b in om.buckets(cfg):                          # buckets tile the parameter list in order
        assert b == list(range(b[0], b[-1] + 1))
    n = wl.n_params(cfg)
    e = 4 if cfg.dtype == "fp32" else 2
    shard = [4, 4] + ([] if cfg.dtype == "fp32" else [4])      # m, v, master: 1/world each
    C = om.persistent_bytes(cfg, cfg.n_seqs, cfg.max_seq, world, True)
    C1 = om.persistent_bytes(cfg, cfg.n_seqs, cfg.max_seq)
    fixed = C1 - a16(om.padded_numel(cfg) * (e + 4 + sum(shard)))   # batch buffers, workspaces
    assert C == a16(npad * e) + a16(npad * 4) + sum(a16(npad // world * s) for s in shard) + fixed
    if world == 1:
        assert C == C1                                 # no padding change at one rank
    if cfg.dtype == "bf16":                            # 18 B/param -> 6 + 12/world B/param
        per = (C - fixed) / n
        assert abs(per - (6 + 12 / world)) < 0.01 * (6 + 12 / world)


@pytest.mark.parametrize("name", CFGS)
@pytest.mark.parametrize("world", [2, 8])
def test_zero1_library_accounting_matches_oracle(name, world):
    """Host-only context of rank 0 of `world`: C, dry-run peaks and collector
    samples equal the oracle's ZeRO-1 event model; plans under the non-sharded
    bench budget never drop more layers than without ZeRO-1."""
    cfg = wl.CONFIGS[name]
    szmax = om.sizes(cfg, cfg.n_seqs, cfg.max_seq)
    M = max(szmax.C + int(cfg.budget_frac * (om.no_ckpt_peak(szmax) - szmax.C)), om.lower_bound(szmax))
    ctx = mb.Mimose(cfg, M, world=world, zero1=1)
    assert ctx.stats()["persistent_bytes"] == om.persistent_bytes(cfg, cfg.n_seqs, cfg.max_seq, world, True)
    for S in sorted({cfg.seq_lo, cfg.max_seq}):
        S = wl.roundup(S, cfg.pad)
        sz = om.sizes(cfg, cfg.n_seqs, S, world=world, zero1=True)
        assert ctx.dry_run(cfg.n_seqs, S, []) == om.no_ckpt_peak(sz)
        assert ctx.dry_run(cfg.n_seqs, S, range(cfg.n_layers)) == om.lower_bound(sz)
        got = ctx.dry_collect(cfg.n_seqs, S)
        want = om.collect_samples(sz)
        for k in ("C", "E", "Hd", "Th", "Tb", "Te", "a", "y"):
            assert got[k] == want[k]
        st0, d0, _ = op.plan(om.collect_samples(om.sizes(cfg, cfg.n_seqs, S)), M)
        st1, d1, pk1 = op.plan(want, M)
        assert st1 == op.OK and pk1 <= M
        assert st0 != op.OK or len(d1) <= len(d0)
    ctx.close()
