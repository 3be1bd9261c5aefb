"""Encoder-decoder on the B200 (reading A32), through the C ABI:

* loss and every gradient against the fp64 oracle (encdec_step_grads) under
  SURVEY c-K's metric (tests/parity_metrics.py), at reduced and at full width;
* bit-exact recompute replay: plans over the encoder + decoder units give the
  no-checkpoint step's loss and gradients bitwise;
* the sheltered phase on 2-D keys: samples == the oracle event model, plans ==
  the oracle planner on its bivariate estimator, arena peak == simulator <= M.
"""
import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from oracle import estimator as oe
from oracle import memsim as om
from oracle import model as omodel
from oracle import planner as op
from paper_conf_ipps_liaolysshfyctzlq23_b200 import workload as wl

import parity_metrics as pm

SMALL = wl.small_config("t5-base", n_layers=2, n_dec_layers=2, hidden=128, heads=2, ffn=256, vocab=500,
                        max_pos=128, n_seqs=4, seq_lo=17, seq_hi=100, pad=8)
LONG = wl.small_config("t5-base", n_layers=2, n_dec_layers=2, hidden=128, heads=2, ffn=256, vocab=500,
                       max_pos=512, n_seqs=3, seq_lo=130, seq_hi=300, pad=8)      # tiled cross-attention
FULL = wl.small_config("t5-base", n_layers=2, n_dec_layers=2)


def mb():
    from paper_conf_ipps_liaolysshfyctzlq23_b200 import binding
    return binding


def peak_max(cfg):
    sz = om.sizes_encdec(cfg, cfg.n_seqs, cfg.max_seq, cfg.max_seq)
    return om.simulate_step_encdec(sz, []).peak


def make_ctx(cfg, budget=None, **kw):
    budget = budget or peak_max(cfg)
    slab = torch.empty(budget, dtype=torch.uint8, device="cuda")
    ctx = mb().Mimose(cfg, budget, slab=slab, stream=torch.cuda.current_stream(), **kw)
    ctx._slab_keep = slab
    return ctx


def step(ctx, b, plan=()):
    p = mb().Plan()
    p.drop_mask = sum(1 << u for u in plan)
    loss = ctx.forward(ctx.host_batch(b), p)
    ctx.backward()
    torch.cuda.synchronize()
    return loss, ctx.get_grads()


def bf16(params):
    return {k: torch.tensor(v).bfloat16().double().numpy() for k, v in params.items()}


@pytest.mark.parametrize("name,cfg,S", [("t5-small", SMALL, 100), ("t5-long", LONG, 290), ("t5-s128", FULL, 128),
                                        ("t5-s460", FULL, 460)])
def test_encdec_parity_against_oracle(name, cfg, S):
    params = wl.init_params(cfg, parity=True, seed=11)
    ctx = make_ctx(cfg)
    ctx.set_params(wl.pack_params(cfg, params))
    b = wl.make_batch(cfg, S, seed=5)
    loss, g = step(ctx, b, [0, 2])
    ref_loss, G = omodel.train_step_grads(cfg, bf16(params), b, wl.dropout_seed(cfg), ctx.stats()["steps"])
    pm.check(name, cfg, wl.unpack_params(cfg, g), G, loss, ref_loss)
    ctx.close()


@pytest.mark.parametrize("cfg,S", [(SMALL, 77), (LONG, 250)])
def test_encdec_recompute_replay_bitwise(cfg, S):
    params = wl.init_params(cfg, parity=True, seed=3)
    b = wl.make_batch(cfg, S, seed=7)
    ref = None
    n = cfg.n_layers + cfg.n_dec_layers
    for plan in ([], [0], [2], list(range(n)), [1, 3], [n - 1]):
        ctx = make_ctx(cfg)
        ctx.set_params(wl.pack_params(cfg, params))
        loss, g = step(ctx, b, plan)
        st = ctx.stats()
        assert st["peak_bytes"] == om.simulate_step_encdec(
            om.sizes_encdec(cfg, cfg.n_seqs, b.seq_len, b.dec_len), plan).peak
        ctx.close()
        if ref is None:
            ref = (loss, g)
        else:
            assert loss == ref[0] and np.array_equal(g, ref[1]), plan


def test_encdec_collector_plans_and_budget():
    cfg = SMALL
    szmax = om.sizes_encdec(cfg, cfg.n_seqs, cfg.max_seq, cfg.max_seq)
    n = cfg.n_layers + cfg.n_dec_layers
    P0, LB = om.simulate_step_encdec(szmax, []).peak, om.simulate_step_encdec(szmax, range(n)).peak
    M = max(szmax.C + int(0.5 * (P0 - szmax.C)), LB)
    ctx = make_ctx(cfg, M)
    ctx.set_params(wl.pack_params(cfg, wl.init_params(cfg)))
    rng = np.random.default_rng(4)
    i = 0
    while ctx.phase == mb().PHASE_SHELTERED:
        b = wl.make_batch(cfg, int(rng.integers(cfg.seq_lo, cfg.seq_hi + 1)), seed=i)
        ctx.collect(ctx.host_batch(b))
        ctx.backward()
        ctx.step(1e-4)
        i += 1
    samples = []
    for j in range(ctx.stats()["n_samples"]):
        s = ctx.sample(j)
        want = om.collect_samples_encdec(om.sizes_encdec(cfg, cfg.n_seqs, s["x"] // cfg.n_seqs, s["xt"] // cfg.n_seqs))
        for k in ("C", "E", "Hd", "Th", "Tb", "Te", "a", "y"):
            assert s[k] == want[k], k
        assert all(t > 0 for t in s["t_ms"][:n])
        want["x"], want["xt"] = s["x"], s["xt"]
        samples.append(want)
    est = oe.Estimator2D(samples)
    for k in range(20):
        b = wl.make_batch(cfg, int(rng.integers(cfg.seq_lo, cfg.seq_hi + 1)), seed=1000 + k)
        x, xt = b.input_size2
        p = ctx.plan(x, xt)
        ost, od, _ = op.plan(est.predict(x, xt), M)
        assert p.dropped == list(od)
        loss = ctx.forward(ctx.host_batch(b), p)
        ctx.backward()
        ctx.step(1e-4)
        st = ctx.stats()
        assert st["peak_bytes"] == om.simulate_step_encdec(
            om.sizes_encdec(cfg, cfg.n_seqs, b.seq_len, b.dec_len), p.dropped).peak <= M
        assert np.isfinite(loss)
    assert ctx.stats()["violations"] == 0
    ctx.close()
