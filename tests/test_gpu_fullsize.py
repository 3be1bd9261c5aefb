"""Full-size parity: full hidden width, heads, FFN width and vocabulary of every
GPU BASELINE config, at its S_max, in the launch configuration bench.py times
(tcgen05 GEMMs and attention), with 2-3 layers so the fp64 oracle finishes:

* loss and every gradient tensor against the fp64 oracle under SURVEY c-K's
  metric (tests/parity_metrics.py): the per-tensor normwise inf-norm error
  max|g - g_ref| / max|g_ref| <= 2e-2 (bf16), exceeded only where the
  bf16-storage emulation shows the excess is inherent; provably zero tensors
  (MC classifier bias, QA bias, last LN2 shift) at fp32 round-off
* bit-exact recompute replay: a plan dropping layers vs no checkpointing
* the arena peak equals the oracle event model and is <= the budget
* BERT-base at the full 12 layers too, at the bench budget (the plan
  Algorithm 1 gives there), ragged S_pad = 40

Each case writes its per-tensor error table to gpurun_out/parity/ (the
committed summary is profiles/r2/parity_tables.md).
"""
import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = [pytest.mark.gpu, pytest.mark.slow]

from oracle import memsim as om
from oracle import model as omodel
from oracle import planner as op
from paper_conf_ipps_liaolysshfyctzlq23_b200 import workload as wl

import parity_metrics as pm

FULL = {
    # BERT-base, SWAG-like MC (64 sequences = 16 questions x 4), S_max = 128
    "bb-s128": (wl.small_config("bert-base", n_layers=3), 128, [0, 1]),
    # BERT-large, SQuAD-like QA (12 sequences), S_max = 512
    "bl-s512": (wl.small_config("bert-large", n_layers=2), 512, [0]),
    # RoBERTa-large MC, S_max = 512 (16 sequences = 4 questions: bounds the fp64 oracle's RAM)
    "rl-s512": (wl.small_config("roberta-large", n_layers=2, n_seqs=16), 512, [0]),
    # heterogeneous stages: BERT-base width, one layer per stage, FFN 4096 / 3072 / 1536
    "hetero-s128": (wl.small_config("hetero", n_layers=3, ffn_layers=(4096, 3072, 1536)), 128, [0, 1]),
    # GPT-2 medium, causal, tied 50257-word LM head, S_max = 1024 (2 sequences)
    "g2-s1024": (wl.small_config("gpt2-medium", n_layers=2, n_seqs=2), 1024, [1]),
}


def run(cfg, b, budget, slab_bytes, mask, params, enforce=1, **kw):
    from paper_conf_ipps_liaolysshfyctzlq23_b200 import binding as mb
    slab = torch.empty(slab_bytes, dtype=torch.uint8, device="cuda")
    ctx = mb.Mimose(cfg, budget, slab=slab, stream=torch.cuda.current_stream(), enforce_budget=enforce, **kw)
    ctx.set_params(wl.pack_params(cfg, params))
    p = mb.Plan()
    p.drop_mask = mask
    loss = ctx.forward(ctx.host_batch(b), p)
    ctx.backward()
    torch.cuda.synchronize()
    g = ctx.get_grads()
    st = ctx.stats()
    ctx.close()
    return loss, g, st


def emulator(cfg, W, b):
    if cfg.arch != wl.ARCH_POST_LN:
        return None
    import bf16_emulation as be
    return lambda: be.train_step_grads(cfg, W, b, wl.dropout_seed(cfg), 1, gelu="tanh")


def bf16_weights(params):
    return {k: torch.tensor(v).bfloat16().double().numpy() for k, v in params.items()}


@pytest.mark.parametrize("case", list(FULL))
def test_full_width_parity_at_smax(case):
    cfg, S, dropped = FULL[case]
    params = wl.init_params(cfg, parity=True, seed=11)
    b = wl.make_batch(cfg, S, seed=5)
    assert b.seq_len == S == cfg.max_seq
    sz = om.sizes(cfg, cfg.n_seqs, S)
    P0 = om.no_ckpt_peak(sz)
    mask = sum(1 << l for l in dropped)
    pk = om.peak(sz, dropped)
    loss, g, st = run(cfg, b, pk, pk, mask, params)           # budget = exactly the plan's peak
    assert st["peak_bytes"] == pk and st["violations"] == 0
    loss0, g0, _ = run(cfg, b, P0, P0, 0, params)
    assert loss == loss0 and np.array_equal(g, g0)            # recompute replay is bit-exact
    W = bf16_weights(params)
    ref_loss, G = omodel.train_step_grads(cfg, W, b, wl.dropout_seed(cfg), 1)
    pm.check(case, cfg, wl.unpack_params(cfg, g), G, loss, ref_loss, emulator(cfg, W, b))


def test_bert_base_full_depth_bench_budget():
    """All 12 layers, BERT init (the weights bench.py trains), the bench's 60%
    budget and the plan Algorithm 1 gives there; ragged batch (S_pad = 40)."""
    cfg = wl.CONFIGS["bert-base"]
    szmax = om.sizes(cfg, cfg.n_seqs, cfg.max_seq)
    M = max(szmax.C + int(cfg.budget_frac * (om.no_ckpt_peak(szmax) - szmax.C)), om.lower_bound(szmax))
    params = wl.init_params(cfg)
    b = wl.make_batch(cfg, 37, seed=5)
    sz = om.sizes(cfg, cfg.n_seqs, b.seq_len)
    status, dropped, _ = op.plan(om.collect_samples(sz), M)
    assert status == op.OK
    mask = sum(1 << l for l in dropped)
    loss_m, g_m, st_m = run(cfg, b, M, M, mask, params)
    assert st_m["peak_bytes"] == om.peak(sz, dropped) <= M
    loss_n, g_n, _ = run(cfg, b, M, om.no_ckpt_peak(szmax) + (1 << 20), 0, params, enforce=0)
    assert loss_m == loss_n and np.array_equal(g_m, g_n)
    W = bf16_weights(params)
    ref_loss, G = omodel.train_step_grads(cfg, W, b, wl.dropout_seed(cfg), 1)
    pm.check("bb-l12-s40-bench", cfg, wl.unpack_params(cfg, g_m), G, loss_m, ref_loss, emulator(cfg, W, b))
