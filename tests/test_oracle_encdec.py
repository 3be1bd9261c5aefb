"""Pins for the encoder-decoder oracle (oracle/model.py
encdec_step_grads; Table II TR-T5, reading A32):

* central finite differences in fp64 (masks held fixed) on every tensor;
* torch CPU fp64 autograd -- an independent re-implementation with
  torch.nn.functional (pre-LN encoder, final LN, pre-LN decoder with causal
  self-attention and cross-attention, tied LM head) with the oracle's dropout
  masks injected -- loss and every gradient within 1e-10 normwise;
* checkpoint identity (c-C): any plan over the encoder + decoder layers gives
  the plain step's loss and gradients bit for bit;
* the dropout sites of the 2 x L layers, the decoder embedding and the two
  cross-attention kinds never collide.
"""
import math

import numpy as np
import pytest
import torch

from oracle import model as om
from oracle import philox as px
from paper_conf_ipps_liaolysshfyctzlq23_b200 import workload as wl


def tiny(**kw):
    base = dict(n_layers=2, n_dec_layers=2, hidden=16, heads=2, ffn=32, vocab=40, max_pos=24, n_seqs=3,
                seq_lo=3, seq_hi=9, pad=1, first_tok=3)
    base.update(kw)
    return wl.small_config("t5-base", **base)


def setup(S=7, seed=5, **kw):
    cfg = tiny(**kw)
    params = wl.init_params(cfg, parity=True, seed=seed)
    batch = wl.make_batch(cfg, S, seed=seed + 1)
    return cfg, params, batch


def torch_step(cfg, params, batch, mk):
    W = {k: torch.tensor(v, dtype=torch.float64, requires_grad=True) for k, v in params.items()}
    F_ = torch.nn.functional
    B, Ss = batch.input_ids.shape
    St = batch.dec_len
    H, h = cfg.hidden, cfg.heads
    d = H // h
    t = lambda a: torch.tensor(a)

    def attn(q, k, v, qS, kS, kvalid, causal, pm):
        q = q.reshape(B, qS, h, d).permute(0, 2, 1, 3)
        k = k.reshape(B, kS, h, d).permute(0, 2, 1, 3)
        v = v.reshape(B, kS, h, d).permute(0, 2, 1, 3)
        s = q @ k.transpose(-1, -2) / math.sqrt(d)
        allowed = kvalid[:, None, None, :].expand(B, h, qS, kS)
        if causal:
            allowed = allowed & torch.tril(torch.ones(qS, kS, dtype=torch.bool))[None, None]
        s = s.masked_fill(~allowed, float("-inf"))
        return ((torch.softmax(s, -1) * t(pm)) @ v).permute(0, 2, 1, 3).reshape(B * qS, H)

    ln = lambda x, p: F_.layer_norm(x, (H,), W[p + ".g"], W[p + ".b"], cfg.ln_eps)
    svalid = torch.arange(Ss)[None, :] < t(batch.lengths)[:, None]
    tvalid = torch.arange(St)[None, :] < t(batch.dec_lengths)[:, None]
    ids = t(batch.input_ids).long().reshape(-1)
    x = (W["emb.word"][ids] + W["emb.pos"][torch.arange(Ss).repeat(B)]) * t(mk.enc.emb())
    for l in range(cfg.n_layers):
        p = f"layer{l}."
        a = ln(x, p + "ln1")
        qkv = F_.linear(a, W[p + "qkv.w"], W[p + "qkv.b"])
        o = attn(qkv[:, :H], qkv[:, H:2 * H], qkv[:, 2 * H:], Ss, Ss, svalid, False, mk.enc.attn_probs(l))
        x = x + F_.linear(o, W[p + "o.w"], W[p + "o.b"]) * t(mk.enc.attn_out(l))
        m = ln(x, p + "ln2")
        g = F_.gelu(F_.linear(m, W[p + "f1.w"], W[p + "f1.b"]), approximate="tanh")
        x = x + F_.linear(g, W[p + "f2.w"], W[p + "f2.b"]) * t(mk.enc.ffn_out(l))
    enc = ln(x, "enc.lnf")
    tids = t(batch.dec_ids).long().reshape(-1)
    y = (W["emb.word"][tids] + W["emb.pos"][torch.arange(St).repeat(B)]) * t(mk.dec_emb())
    for j in range(cfg.n_dec_layers):
        p, L = f"dec{j}.", cfg.n_layers + j
        a = ln(y, p + "ln1")
        qkv = F_.linear(a, W[p + "qkv.w"], W[p + "qkv.b"])
        o = attn(qkv[:, :H], qkv[:, H:2 * H], qkv[:, 2 * H:], St, St, tvalid, True, mk.dec.attn_probs(L))
        y = y + F_.linear(o, W[p + "o.w"], W[p + "o.b"]) * t(mk.dec.attn_out(L))
        c = ln(y, p + "ln2")
        q = F_.linear(c, W[p + "cq.w"], W[p + "cq.b"])
        kv = F_.linear(enc, W[p + "ckv.w"], W[p + "ckv.b"])
        oc = attn(q, kv[:, :H], kv[:, H:], St, Ss, svalid, False, mk.cross_probs(L))
        y = y + F_.linear(oc, W[p + "co.w"], W[p + "co.b"]) * t(mk.cross_out(L))
        m = ln(y, p + "ln3")
        g = F_.gelu(F_.linear(m, W[p + "f1.w"], W[p + "f1.b"]), approximate="tanh")
        y = y + F_.linear(g, W[p + "f2.w"], W[p + "f2.b"]) * t(mk.dec.ffn_out(L))
    logits = ln(y, "lnf") @ W["emb.word"].T
    rows, tg = [], []
    for b in range(B):
        n = int(batch.dec_lengths[b])
        for s in range(n - 1):
            rows.append(b * St + s)
            tg.append(int(batch.dec_ids[b, s + 1]))
    loss = F_.cross_entropy(logits[rows], torch.tensor(tg))
    loss.backward()
    return float(loss), {k: w.grad.numpy() for k, w in W.items()}


def test_torch_autograd_agrees():
    cfg, params, batch = setup()
    seed, step = 21, 4
    loss, G = om.train_step_grads(cfg, params, batch, seed, step)
    B, Ss = batch.input_ids.shape
    mk = om.EncDecMasks(cfg, B, Ss, batch.dec_len, seed, step)
    tl, TG = torch_step(cfg, {k: v.astype(np.float64) for k, v in params.items()}, batch, mk)
    assert abs(loss - tl) <= 1e-12 * max(1.0, abs(tl))
    for k in TG:
        sc = max(float(np.abs(TG[k]).max()), 1e-6)
        assert np.abs(G[k] - TG[k]).max() / sc <= 1e-10, k


def test_finite_differences():
    cfg, params, batch = setup(S=6, seed=8)
    seed, step = 3, 2
    loss, G = om.train_step_grads(cfg, params, batch, seed, step)
    P = {k: v.astype(np.float64) for k, v in params.items()}
    rng = np.random.default_rng(1)
    h = 1e-6
    for name, g in G.items():
        flat = P[name].reshape(-1)
        idx = rng.choice(flat.size, size=min(4, flat.size), replace=False)
        num = []
        for i in idx:
            old = flat[i]
            flat[i] = old + h
            lp, _ = om.train_step_grads(cfg, P, batch, seed, step)
            flat[i] = old - h
            lm, _ = om.train_step_grads(cfg, P, batch, seed, step)
            flat[i] = old
            num.append((lp - lm) / (2 * h))
        scale = max(np.abs(g).max(), 1e-12)
        assert np.abs(np.array(num) - g.reshape(-1)[idx]).max() <= 1e-6 * scale + 2e-9, name


def test_checkpoint_identity():
    cfg, params, batch = setup()
    ref = om.train_step_grads(cfg, params, batch, 9, 1)
    for plan in ([0], [2, 3], [0, 1, 2, 3], [1, 3]):
        got = om.train_step_grads(cfg, params, batch, 9, 1, plan=plan)
        assert got[0] == ref[0]
        for k in ref[1]:
            assert np.array_equal(got[1][k], ref[1][k]), (plan, k)


def test_dropout_sites_distinct():
    cfg = wl.CONFIGS["t5-base"]
    seen = set()
    L = cfg.n_layers + cfg.n_dec_layers
    for layer in list(range(L)) + [px.LAYER_NONE, om.DEC_EMB]:
        for kind in range(7):
            w = px.site_word(kind, layer)
            assert w not in seen
            seen.add(w)
