"""Pins for oracle/model.py (CPU).

* central finite differences in fp64 (masks held fixed) -> every gradient path
* torch CPU fp64 autograd (an independent library) with the oracle's masks
  injected -> loss and every gradient, normwise <= 1e-10
* checkpoint identity (c-C): plan-driven execution is bitwise the plain step
* per-op closed forms (softmax rows, LN moments, GELU values)
* AdamW against torch.optim.AdamW in fp64
"""
import math

import numpy as np
import pytest
import torch

from oracle import model as om
from oracle import philox as px
from paper_conf_ipps_liaolysshfyctzlq23_b200 import workload as wl


def tiny(head, **kw):
    base = dict(n_layers=2, hidden=16, heads=2, ffn=32, vocab=40, max_pos=16,
                first_tok=3, cls_id=1, sep_id=2, pad_id=0, n_seqs=4, seq_lo=3,
                seq_hi=7, pad=1, n_choices=2, n_labels=3, head=head)
    base.update(kw)
    return wl.small_config("toy", **base)


HEADS = [wl.HEAD_SEQCLS, wl.HEAD_MC, wl.HEAD_QA]


def setup(head, S=6, seed=5, **kw):
    cfg = tiny(head, **kw)
    params = wl.init_params(cfg, parity=True, seed=seed)
    batch = wl.make_batch(cfg, S, seed=seed + 1)
    return cfg, params, batch


def normwise(a, b, floor=1e-6):
    """max|a-b| / max|b|; the floor keeps identically-zero gradients (e.g. the
    last LN shift under the QA head, whose logit gradients sum to zero) from
    dividing round-off by round-off."""
    a, b = np.asarray(a, np.float64), np.asarray(b, np.float64)
    den = max(float(np.abs(b).max()), floor)
    return float(np.abs(a - b).max() / den)


# ------------------------------------------------------------------ FD -----

@pytest.mark.parametrize("head", HEADS)
def test_finite_differences(head):
    cfg, params, batch = setup(head)
    seed, step = 11, 3
    loss, G = om.train_step_grads(cfg, params, batch, seed, step)
    P = {k: v.astype(np.float64) for k, v in params.items()}
    rng = np.random.default_rng(0)
    h = 1e-6
    for name, g in G.items():
        flat = P[name].reshape(-1)
        idx = rng.choice(flat.size, size=min(6, flat.size), replace=False)
        num = np.empty(idx.size)
        for j, i in enumerate(idx):
            old = flat[i]
            flat[i] = old + h
            lp, _ = om.train_step_grads(cfg, P, batch, seed, step)
            flat[i] = old - h
            lm, _ = om.train_step_grads(cfg, P, batch, seed, step)
            flat[i] = old
            num[j] = (lp - lm) / (2 * h)
        ana = g.reshape(-1)[idx]
        scale = max(np.abs(g).max(), 1e-12)
        # FD round-off floor: eps_64 * |loss| / h ~ 2e-10
        assert np.abs(num - ana).max() <= 1e-6 * scale + 2e-9, name


# ------------------------------------------------------- torch autograd -----

def torch_step(cfg, params, batch, masks):
    """Independent re-implementation with torch.nn.functional (fp64)."""
    W = {k: torch.tensor(v, dtype=torch.float64, requires_grad=True) for k, v in params.items()}
    B, S = batch.input_ids.shape
    H, h = cfg.hidden, cfg.heads
    d = H // h
    F_ = torch.nn.functional
    ids = torch.tensor(batch.input_ids, dtype=torch.long)
    tt = torch.tensor(batch.token_type, dtype=torch.long)
    pos = torch.arange(S) + cfg.pos_offset
    z = W["emb.word"][ids] + W["emb.pos"][pos][None] + W["emb.type"][tt]
    x = F_.layer_norm(z, (H,), W["emb.ln.g"], W["emb.ln.b"], cfg.ln_eps)
    x = x.reshape(B * S, H) * torch.tensor(masks.emb())
    valid = torch.arange(S)[None, :] < torch.tensor(batch.lengths)[:, None]
    for l in range(cfg.n_layers):
        p = f"layer{l}."
        qkv = F_.linear(x, W[p + "qkv.w"], W[p + "qkv.b"]).reshape(B, S, 3, h, d)
        q, k, v = (qkv[:, :, i].permute(0, 2, 1, 3) for i in range(3))
        s = q @ k.transpose(-1, -2) / math.sqrt(d)
        s = s.masked_fill(~valid[:, None, None, :], float("-inf"))
        pr = torch.softmax(s, dim=-1) * torch.tensor(masks.attn_probs(l))
        o = (pr @ v).permute(0, 2, 1, 3).reshape(B * S, H)
        z1 = x + F_.linear(o, W[p + "o.w"], W[p + "o.b"]) * torch.tensor(masks.attn_out(l))
        h1 = F_.layer_norm(z1, (H,), W[p + "ln1.g"], W[p + "ln1.b"], cfg.ln_eps)
        g = F_.gelu(F_.linear(h1, W[p + "f1.w"], W[p + "f1.b"]))
        z2 = h1 + F_.linear(g, W[p + "f2.w"], W[p + "f2.b"]) * torch.tensor(masks.ffn_out(l))
        x = F_.layer_norm(z2, (H,), W[p + "ln2.g"], W[p + "ln2.b"], cfg.ln_eps)
    if cfg.head in (wl.HEAD_SEQCLS, wl.HEAD_MC):
        c = x.reshape(B, S, H)[:, 0]
        pl = torch.tanh(F_.linear(c, W["pool.w"], W["pool.b"])) * torch.tensor(masks.head())
        logits = F_.linear(pl, W["cls.w"], W["cls.b"])
        if cfg.head == wl.HEAD_MC:
            logits = logits.reshape(B // cfg.n_choices, cfg.n_choices)
        loss = F_.cross_entropy(logits, torch.tensor(batch.labels, dtype=torch.long))
    else:
        lg = F_.linear(x, W["qa.w"], W["qa.b"]).reshape(B, S, 2)
        lg = lg.masked_fill(~valid[:, :, None], float("-inf"))
        lab = torch.tensor(batch.labels, dtype=torch.long)
        loss = 0.5 * (F_.cross_entropy(lg[:, :, 0], lab[0::2]) + F_.cross_entropy(lg[:, :, 1], lab[1::2]))
    loss.backward()
    return float(loss), {k: t.grad.numpy() for k, t in W.items()}


@pytest.mark.parametrize("head", HEADS)
@pytest.mark.parametrize("p", [0.0, 0.1])
def test_against_torch_autograd(head, p):
    cfg, params, batch = setup(head, S=7, seed=9)
    seed, step = 21, 1
    loss, G = om.train_step_grads(cfg, params, batch, seed, step, p=p)
    masks = om.Masks(cfg, *batch.input_ids.shape, seed, step, 0, p)
    tloss, TG = torch_step(cfg, params, batch, masks)
    assert abs(loss - tloss) <= 1e-12 * max(1.0, abs(tloss))
    for k in TG:
        assert normwise(G[k], TG[k]) <= 1e-10, k


def test_bert_layer_shapes_against_torch_larger():
    """Wider config: H=64, 4 heads, S spanning ragged lengths."""
    cfg = tiny(wl.HEAD_MC, hidden=64, heads=4, ffn=128, n_layers=3, n_seqs=6, n_choices=3)
    params = wl.init_params(cfg, parity=True, seed=3)
    batch = wl.make_batch(cfg, 9, seed=4)
    loss, G = om.train_step_grads(cfg, params, batch, 7, 2)
    masks = om.Masks(cfg, *batch.input_ids.shape, 7, 2)
    tloss, TG = torch_step(cfg, params, batch, masks)
    assert abs(loss - tloss) <= 1e-12
    for k in TG:
        assert normwise(G[k], TG[k]) <= 1e-10, k


# --------------------------------------------------- checkpoint identity -----

@pytest.mark.parametrize("plan", [[], [0], [1], [0, 1], [0, 1, 2]])
def test_checkpoint_identity_bitwise(plan):
    cfg = tiny(wl.HEAD_SEQCLS, n_layers=3)
    params = wl.init_params(cfg, parity=True, seed=1)
    batch = wl.make_batch(cfg, 6, seed=2)
    l0, g0 = om.train_step_grads(cfg, params, batch, 5, 0)
    l1, g1 = om.train_step_grads(cfg, params, batch, 5, 0, plan=plan)
    assert l0 == l1
    for k in g0:
        assert np.array_equal(g0[k], g1[k]), k


# ------------------------------------------------------------- closed forms -----

def test_softmax_rows_and_layernorm_moments():
    rng = np.random.default_rng(0)
    s = rng.normal(size=(5, 9))
    p, lse = om.softmax_lastdim(s)
    assert np.allclose(p.sum(-1), 1.0, atol=1e-15)
    assert np.allclose(lse, np.log(np.exp(s).sum(-1)), atol=1e-13)
    z = rng.normal(3, 2, size=(7, 32))
    y, (xhat, rstd) = om.layernorm(z, np.ones(32), np.zeros(32), 1e-12)
    assert np.allclose(y.mean(-1), 0, atol=1e-14)
    assert np.allclose((y * y).mean(-1), 1, atol=1e-10)


def test_gelu_values():
    assert om.gelu(np.array([0.0]))[0] == 0.0
    # GELU(1) = Phi(1) = 0.8413447460685429... (standard normal CDF)
    assert abs(om.gelu(np.array([1.0]))[0] - 0.8413447460685429) < 1e-15
    assert abs(om.gelu(np.array([-1.0]))[0] + (1 - 0.8413447460685429)) < 1e-15
    u = np.linspace(-4, 4, 17)
    fd = (om.gelu(u + 1e-6) - om.gelu(u - 1e-6)) / 2e-6
    assert np.abs(om.gelu_bwd(np.ones_like(u), u) - fd).max() < 1e-8


def test_dropout_masks_documented_layout():
    cfg = tiny(wl.HEAD_SEQCLS)
    m = om.Masks(cfg, 2, 5, seed=123, step=4)
    a = m.attn_probs(1)
    words = px.uniform_words(2 * cfg.heads * 5 * 5, 123, px.site_word(px.KIND_ATTN_PROBS, 1), 4)
    keep = words < px.keep_threshold(0.1)
    assert np.array_equal((a > 0).reshape(-1), keep)
    assert np.allclose(a[a > 0], 1 / 0.9)


# ------------------------------------------------------------------ AdamW -----

def test_adamw_against_torch():
    rng = np.random.default_rng(1)
    shapes = {"a": (4, 3), "b": (5,)}
    P = {k: rng.normal(size=s) for k, s in shapes.items()}
    m = {k: np.zeros(s) for k, s in shapes.items()}
    v = {k: np.zeros(s) for k, s in shapes.items()}
    tp = {k: torch.tensor(P[k], requires_grad=True) for k in P}
    opt = torch.optim.AdamW(list(tp.values()), lr=1e-2, betas=(0.9, 0.999), eps=1e-8, weight_decay=0.01)
    for t in range(1, 4):
        G = {k: rng.normal(size=s) for k, s in shapes.items()}
        for k in tp:
            tp[k].grad = torch.tensor(G[k])
        opt.step()
        P, m, v = om.adamw(P, G, m, v, t, 1e-2, wd=0.01)
        for k in P:
            assert np.allclose(P[k], tp[k].detach().numpy(), rtol=0, atol=1e-14)


# ------------------------------------------------------------ GPT-2 (pre-LN) --

def tiny_gpt2(**kw):
    base = dict(n_layers=2, hidden=16, heads=2, ffn=32, vocab=50, max_pos=16, pad_id=49, cls_id=49,
                sep_id=49, first_tok=0, n_seqs=3, seq_lo=3, seq_hi=9, pad=1)
    base.update(kw)
    return wl.small_config("gpt2-medium", **base)


def torch_step_gpt2(cfg, params, batch, masks):
    """Independent GPT-2 (pre-LN, causal, tied LM head, tanh-GELU) in torch fp64."""
    W = {k: torch.tensor(v, dtype=torch.float64, requires_grad=True) for k, v in params.items()}
    B, S = batch.input_ids.shape
    H, h = cfg.hidden, cfg.heads
    d = H // h
    F_ = torch.nn.functional
    ids = torch.tensor(batch.input_ids, dtype=torch.long)
    x = (W["emb.word"][ids] + W["emb.pos"][torch.arange(S)][None]).reshape(B * S, H) * torch.tensor(masks.emb())
    valid = torch.arange(S)[None, :] < torch.tensor(batch.lengths)[:, None]
    causal = torch.arange(S)[None, :] <= torch.arange(S)[:, None]
    allowed = valid[:, None, None, :] & causal[None, None]
    for l in range(cfg.n_layers):
        p = f"layer{l}."
        a = F_.layer_norm(x, (H,), W[p + "ln1.g"], W[p + "ln1.b"], cfg.ln_eps)
        qkv = F_.linear(a, W[p + "qkv.w"], W[p + "qkv.b"]).reshape(B, S, 3, h, d)
        q, k, v = (qkv[:, :, i].permute(0, 2, 1, 3) for i in range(3))
        sc = (q @ k.transpose(-1, -2) / math.sqrt(d)).masked_fill(~allowed, float("-inf"))
        pr = torch.softmax(sc, dim=-1) * torch.tensor(masks.attn_probs(l))
        o = (pr @ v).permute(0, 2, 1, 3).reshape(B * S, H)
        r1 = x + F_.linear(o, W[p + "o.w"], W[p + "o.b"]) * torch.tensor(masks.attn_out(l))
        m = F_.layer_norm(r1, (H,), W[p + "ln2.g"], W[p + "ln2.b"], cfg.ln_eps)
        g = F_.gelu(F_.linear(m, W[p + "f1.w"], W[p + "f1.b"]), approximate="tanh")
        x = r1 + F_.linear(g, W[p + "f2.w"], W[p + "f2.b"]) * torch.tensor(masks.ffn_out(l))
    hf = F_.layer_norm(x, (H,), W["lnf.g"], W["lnf.b"], cfg.ln_eps)
    logits = (hf @ W["emb.word"].t()).reshape(B, S, -1)
    labels = ids.clone()
    labels[~valid] = -100
    loss = F_.cross_entropy(logits[:, :-1].reshape(-1, cfg.vocab), labels[:, 1:].reshape(-1), ignore_index=-100)
    loss.backward()
    return float(loss), {k: t.grad.numpy() for k, t in W.items()}


@pytest.mark.parametrize("p", [0.0, 0.1])
def test_gpt2_against_torch_autograd(p):
    cfg = tiny_gpt2()
    params = wl.init_params(cfg, parity=True, seed=4)
    batch = wl.make_batch(cfg, 8, seed=6)
    loss, G = om.train_step_grads(cfg, params, batch, 13, 2, p=p)
    masks = om.Masks(cfg, *batch.input_ids.shape, 13, 2, 0, p)
    tloss, TG = torch_step_gpt2(cfg, params, batch, masks)
    assert abs(loss - tloss) <= 1e-12 * max(1.0, abs(tloss))
    for k in TG:
        assert normwise(G[k], TG[k]) <= 1e-10, k


def test_gpt2_finite_differences_and_replay():
    cfg = tiny_gpt2()
    params = {k: v.astype(np.float64) for k, v in wl.init_params(cfg, parity=True, seed=8).items()}
    batch = wl.make_batch(cfg, 7, seed=2)
    loss, G = om.train_step_grads(cfg, params, batch, 3, 1)
    rng = np.random.default_rng(1)
    for name in ("emb.word", "layer0.qkv.w", "layer1.f2.w", "layer1.ln1.g", "lnf.b", "emb.pos"):
        flat = params[name].reshape(-1)
        for i in rng.choice(flat.size, 4, replace=False):
            old = flat[i]
            flat[i] = old + 1e-6
            lp, _ = om.train_step_grads(cfg, params, batch, 3, 1)
            flat[i] = old - 1e-6
            lm, _ = om.train_step_grads(cfg, params, batch, 3, 1)
            flat[i] = old
            assert abs((lp - lm) / 2e-6 - G[name].reshape(-1)[i]) <= 1e-6 * np.abs(G[name]).max() + 2e-9, name
    for plan in ([0], [0, 1]):
        l2, G2 = om.train_step_grads(cfg, params, batch, 3, 1, plan=plan)
        assert l2 == loss and all(np.array_equal(G[k], G2[k]) for k in G)
