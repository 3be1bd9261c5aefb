"""TEST INFRASTRUCTURE: the fp64 oracle step of a post-LN encoder with every
tensor the bf16 CUDA path STORES in bf16 rounded to bf16 at that point
(reading R-P), everything else exact fp64.  It measures the error
that bf16 storage alone imposes on a correct implementation, so a GPU
gradient whose inf-norm error vs the plain fp64 oracle exceeds SURVEY c-K's
2e-2 can be shown to be inherent (VERDICT r1 "next" item 2).

Storage points (ctx.cpp schedule; DESIGN §3/§5):
  forward   x_l (layer input), QKV, P~ (attention probabilities after dropout,
            the PV operand), O, h1, u, g, y; z1/z2/LN statistics stay fp32
  backward  dt2 = dz2*mask, du = (dt2 W2) * GELU'(u), dt1, dO, dS (the
            dQ/dK operand), dQKV; dh1, dz1 and the inter-layer dy stay fp32;
            the bias gradients of the out-projection and FFN2 sum the stored
            bf16 dt1 / dt2 rows (as the LN-backward kernel's partials do)
  embedding x1 = drop(LN0(z0));  head: pooled
The building blocks are the oracle's own (linear, layernorm, gelu, softmax,
Masks, embed/head); with rnd = identity this function returns the oracle's
result exactly (pinned in tests/test_bf16_emulation.py).
"""
from __future__ import annotations

import math

import numpy as np

from oracle import model as om
from paper_conf_ipps_liaolysshfyctzlq23_b200.workload import ARCH_POST_LN, Batch, ModelConfig


def bf16(a):
    """Round-to-nearest-even to bfloat16, returned as float64."""
    a = np.asarray(a, np.float64)
    f = a.astype(np.float32)
    u = f.view(np.uint32).astype(np.uint64)
    u = (u + 0x7FFF + ((u >> 16) & 1)) & 0xFFFF0000
    return u.astype(np.uint32).view(np.float32).astype(np.float64)


def ident(a):
    return a


def _attn_fwd(qkv, lengths, B, S, h, pmask, r):
    H = qkv.shape[1] // 3
    d = H // h
    sh = lambda t: t.reshape(B, S, h, d).transpose(0, 2, 1, 3)
    q, k, v = sh(qkv[:, :H]), sh(qkv[:, H:2 * H]), sh(qkv[:, 2 * H:])
    s = q @ k.transpose(0, 1, 3, 2) / math.sqrt(d)
    keyvalid = np.arange(S)[None, :] < np.asarray(lengths)[:, None]
    s = np.where(np.broadcast_to(keyvalid[:, None, None, :], s.shape), s, -np.inf)
    p, _ = om.softmax_lastdim(s)
    pd = r(p * pmask)
    o = r(pd @ v)
    return o.transpose(0, 2, 1, 3).reshape(B * S, H), (q, k, v, p, pd, o)


def _attn_bwd(dout, cache, B, S, h, pmask, r):
    q, k, v, p, pd, o = cache
    d = q.shape[-1]
    H = h * d
    do = dout.reshape(B, S, h, d).transpose(0, 2, 1, 3)
    dv = pd.transpose(0, 1, 3, 2) @ do
    dp = (do @ v.transpose(0, 1, 3, 2)) * pmask
    D = (do * o).sum(axis=-1, keepdims=True)          # rowsum(dO o O) = rowsum(dP o P)
    ds = r(p * (dp - D))
    dq = ds @ k / math.sqrt(d)
    dk = ds.transpose(0, 1, 3, 2) @ q / math.sqrt(d)
    flat = lambda t: t.transpose(0, 2, 1, 3).reshape(B * S, H)
    return r(np.concatenate([flat(dq), flat(dk), flat(dv)], axis=1))


def _layer_fwd(cfg, W, l, x, lengths, B, S, masks, r, gelu):
    p = f"layer{l}."
    qkv = r(om.linear(x, W[p + "qkv.w"], W[p + "qkv.b"]))
    o, ac = _attn_fwd(qkv, lengths, B, S, cfg.heads, masks.attn_probs(l), r)
    z1 = x + om.linear(o, W[p + "o.w"], W[p + "o.b"]) * masks.attn_out(l)
    h1f, ln1 = om.layernorm(z1, W[p + "ln1.g"], W[p + "ln1.b"], cfg.ln_eps)
    h1 = r(h1f)
    uf = om.linear(h1, W[p + "f1.w"], W[p + "f1.b"])
    u, g = r(uf), r(gelu[0](uf))
    z2 = h1 + om.linear(g, W[p + "f2.w"], W[p + "f2.b"]) * masks.ffn_out(l)
    y, ln2 = om.layernorm(z2, W[p + "ln2.g"], W[p + "ln2.b"], cfg.ln_eps)
    return r(y), dict(x=x, qkv=qkv, o=o, ac=ac, ln1=ln1, h1=h1, u=u, g=g, ln2=ln2)


def _layer_bwd(cfg, W, l, dy, c, B, S, masks, G, r, gelu):
    p = f"layer{l}."
    dz2, G[p + "ln2.g"], G[p + "ln2.b"] = om.layernorm_bwd(dy, c["ln2"], W[p + "ln2.g"])
    dt2 = r(dz2 * masks.ffn_out(l))
    G[p + "f2.b"] = dt2.sum(axis=0)                     # bias partials sum the stored (bf16) rows
    du = r(gelu[1](dt2 @ W[p + "f2.w"], c["u"]))
    G[p + "f2.w"] = dt2.T @ c["g"]
    dh1, G[p + "f1.w"], G[p + "f1.b"] = om.linear_bwd(du, c["h1"], W[p + "f1.w"])
    dh1 = dh1 + dz2
    dz1, G[p + "ln1.g"], G[p + "ln1.b"] = om.layernorm_bwd(dh1, c["ln1"], W[p + "ln1.g"])
    dt1 = r(dz1 * masks.attn_out(l))
    G[p + "o.b"] = dt1.sum(axis=0)
    do = r(dt1 @ W[p + "o.w"])
    G[p + "o.w"] = dt1.T @ c["o"]
    dqkv = _attn_bwd(do, c["ac"], B, S, cfg.heads, masks.attn_probs(l), r)
    dx, G[p + "qkv.w"], G[p + "qkv.b"] = om.linear_bwd(dqkv, c["x"], W[p + "qkv.w"])
    return dx + dz1


def train_step_grads(cfg: ModelConfig, params, batch: Batch, seed: int, step: int, rnd=bf16,
                     gelu: str = "erf"):
    """Loss and gradients of one plain step with bf16 storage rounding ``rnd``.
    ``gelu="tanh"``: the tanh-form GELU / GELU' that the bf16 tcgen05 epilogues
    evaluate for erf-GELU models (DESIGN reading R-G) instead of the exact erf."""
    gl = (om.gelu, om.gelu_bwd) if gelu == "erf" else (om.gelu_tanh, om.gelu_tanh_bwd)
    assert cfg.arch == ARCH_POST_LN
    W = {k: np.asarray(v, np.float64) for k, v in params.items()}
    B, S = batch.input_ids.shape
    masks = om.Masks(cfg, B, S, seed, step)
    G = {}
    x, ec = om.embed_fwd(cfg, W, batch, masks)
    x = rnd(x)
    caches = []
    for l in range(cfg.n_layers):
        x, c = _layer_fwd(cfg, W, l, x, batch.lengths, B, S, masks, rnd, gl)
        caches.append(c)
    loss, dy = om.head_fwd_bwd(cfg, W, x, batch, masks, G)
    for l in reversed(range(cfg.n_layers)):
        dy = _layer_bwd(cfg, W, l, dy, caches[l], B, S, masks, G, rnd, gl)
    om.embed_bwd(cfg, W, dy, ec, masks, G)
    return loss, G
