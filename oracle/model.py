"""ORACLE (test infrastructure only): fp64 post-LN transformer encoder training step.

What Mimose's training step computes (§II-A: forward -> loss ->
backward -> update; §IV-C P:160 the attention structure Q x K^T -> scale ->
softmax -> x V; P:21 checkpointing = dropping activations and "replaying the
forward computation" in backward).  Checkpointing is exact, so the oracle's
reference result is the PLAIN non-checkpointed step; ``plan`` only changes
what is kept (c-C identity), never the arithmetic.

Model details the paper leaves to HF transformers 4.18 follow reading
R-A24 of DESIGN.md: post-LN BERT/RoBERTa layer, erf-GELU, biased-variance LN,
dropout p on embeddings / attention probabilities / both residual branches /
pooled output, pooler tanh, CE heads.

Every backward formula is textbook backprop written out by hand.
Pinned by: central finite differences (fp64), torch CPU fp64 autograd with the
same masks injected, closed-form per-op identities (tests/test_oracle_model.py).
"""
from __future__ import annotations

import math
from typing import Dict, Optional, Sequence

import numpy as np

from paper_conf_ipps_liaolysshfyctzlq23_b200.workload import (
    ARCH_ENCDEC, ARCH_PRE_LN, HEAD_LM, HEAD_MC, HEAD_QA, HEAD_SEQCLS, Batch, ModelConfig, param_spec)
from . import philox as px


# --------------------------------------------------------------------------
# dropout masks (R-B: element order documented in DESIGN.md)
# --------------------------------------------------------------------------

class Masks:
    """Scaled keep masks m = keep / (1-p) for one step on one rank."""

    def __init__(self, cfg: ModelConfig, B: int, S: int, seed: int, step: int,
                 rank: int = 0, p: Optional[float] = None, override=None):
        self.cfg, self.B, self.S = cfg, B, S
        self.seed, self.step, self.rank = seed, step, rank
        self.p = cfg.p_drop if p is None else p
        self.override = override or {}

    def _mask(self, key, n, kind, layer, shape):
        if key in self.override:
            return self.override[key]
        if self.p <= 0.0:
            return np.ones(shape)
        keep = px.keep_mask(n, self.p, self.seed, px.site_word(kind, layer, self.rank), self.step)
        return keep.reshape(shape).astype(np.float64) / (1.0 - self.p)

    def emb(self):
        T, H = self.B * self.S, self.cfg.hidden
        return self._mask(("emb",), T * H, px.KIND_EMB, px.LAYER_NONE, (T, H))

    def attn_probs(self, l):
        B, S, h = self.B, self.S, self.cfg.heads
        return self._mask(("attn", l), B * h * S * S, px.KIND_ATTN_PROBS, l, (B, h, S, S))

    def attn_out(self, l):
        T, H = self.B * self.S, self.cfg.hidden
        return self._mask(("ao", l), T * H, px.KIND_ATTN_OUT, l, (T, H))

    def ffn_out(self, l):
        T, H = self.B * self.S, self.cfg.hidden
        return self._mask(("fo", l), T * H, px.KIND_FFN_OUT, l, (T, H))

    def head(self):
        B, H = self.B, self.cfg.hidden
        return self._mask(("head",), B * H, px.KIND_HEAD, px.LAYER_NONE, (B, H))


# --------------------------------------------------------------------------
# elementary ops (forward, backward)
# --------------------------------------------------------------------------

def linear(x, w, b):
    """y = x W^T + b."""
    return x @ w.T + b


def linear_bwd(dy, x, w):
    """dx = dy W ; dW = dy^T x ; db = sum_rows dy."""
    return dy @ w, dy.T @ x, dy.sum(axis=0)


def layernorm(z, g, b, eps):
    """(z - mu) / sqrt(var + eps) * g + b, biased variance."""
    mu = z.mean(axis=-1, keepdims=True)
    var = ((z - mu) ** 2).mean(axis=-1, keepdims=True)
    rstd = 1.0 / np.sqrt(var + eps)
    xhat = (z - mu) * rstd
    return xhat * g + b, (xhat, rstd)


def layernorm_bwd(dy, cache, g):
    xhat, rstd = cache
    dg = (dy * xhat).sum(axis=0)
    db = dy.sum(axis=0)
    dxhat = dy * g
    dz = rstd * (dxhat - dxhat.mean(axis=-1, keepdims=True)
                 - xhat * (dxhat * xhat).mean(axis=-1, keepdims=True))
    return dz, dg, db


from scipy.special import erf as _erf   # library primitive (fp64 erf)


def gelu(u):
    """erf-GELU: 0.5 u (1 + erf(u / sqrt 2))."""
    return 0.5 * u * (1.0 + _erf(u / math.sqrt(2.0)))


def gelu_bwd(du_out, u):
    cdf = 0.5 * (1.0 + _erf(u / math.sqrt(2.0)))
    pdf = np.exp(-0.5 * u * u) / math.sqrt(2.0 * math.pi)
    return du_out * (cdf + u * pdf)


_K0 = math.sqrt(2.0 / math.pi)


def gelu_tanh(u):
    """GPT-2 "gelu_new": 0.5 u (1 + tanh(sqrt(2/pi) (u + 0.044715 u^3)))."""
    return 0.5 * u * (1.0 + np.tanh(_K0 * (u + 0.044715 * u ** 3)))


def gelu_tanh_bwd(du_out, u):
    th = np.tanh(_K0 * (u + 0.044715 * u ** 3))
    return du_out * (0.5 * (1.0 + th) + 0.5 * u * (1.0 - th * th) * _K0 * (1.0 + 3 * 0.044715 * u * u))


def softmax_lastdim(s):
    m = s.max(axis=-1, keepdims=True)
    e = np.exp(s - m)
    z = e.sum(axis=-1, keepdims=True)
    return e / z, (m + np.log(z))[..., 0]


def ce_rows(logits, target):
    """mean over rows of -log softmax(logits)[target]; returns loss, dlogits."""
    p, lse = softmax_lastdim(logits)
    n = logits.shape[0]
    loss = float(np.mean(lse - logits[np.arange(n), target]))
    d = p.copy()
    d[np.arange(n), target] -= 1.0
    return loss, d / n


# --------------------------------------------------------------------------
# attention: S = Q K^T / sqrt(d) + key-pad mask, P = softmax, O = drop(P) V
# --------------------------------------------------------------------------

def attention_fwd(qkv, lengths, B, S, h, pmask, causal=False):
    H = qkv.shape[1] // 3
    d = H // h
    q = qkv[:, :H].reshape(B, S, h, d).transpose(0, 2, 1, 3)
    k = qkv[:, H:2 * H].reshape(B, S, h, d).transpose(0, 2, 1, 3)
    v = qkv[:, 2 * H:].reshape(B, S, h, d).transpose(0, 2, 1, 3)
    s = q @ k.transpose(0, 1, 3, 2) / math.sqrt(d)
    keyvalid = np.arange(S)[None, :] < np.asarray(lengths)[:, None]        # [B, S]
    allowed = np.broadcast_to(keyvalid[:, None, None, :], s.shape)
    if causal:                                                             # key k <= query q
        allowed = allowed & (np.arange(S)[None, :] <= np.arange(S)[:, None])[None, None]
    s = np.where(allowed, s, -np.inf)
    p, lse = softmax_lastdim(s)
    pd = p * pmask
    o = pd @ v                                                             # [B,h,S,d]
    out = o.transpose(0, 2, 1, 3).reshape(B * S, H)
    return out, (q, k, v, p, pd, lse)


def attention_bwd(dout, cache, B, S, h, pmask):
    q, k, v, p, pd, _ = cache
    d = q.shape[-1]
    H = h * d
    do = dout.reshape(B, S, h, d).transpose(0, 2, 1, 3)
    dv = pd.transpose(0, 1, 3, 2) @ do
    dpd = do @ v.transpose(0, 1, 3, 2)
    dp = dpd * pmask
    ds = p * (dp - (dp * p).sum(axis=-1, keepdims=True))
    dq = ds @ k / math.sqrt(d)
    dk = ds.transpose(0, 1, 3, 2) @ q / math.sqrt(d)
    def flat(t):
        return t.transpose(0, 2, 1, 3).reshape(B * S, H)
    return np.concatenate([flat(dq), flat(dk), flat(dv)], axis=1)


# --------------------------------------------------------------------------
# encoder layer (post-LN)
# --------------------------------------------------------------------------

def layer_fwd(cfg, W, l, x, lengths, B, S, masks: Masks):
    p = f"layer{l}."
    qkv = linear(x, W[p + "qkv.w"], W[p + "qkv.b"])
    o, acache = attention_fwd(qkv, lengths, B, S, cfg.heads, masks.attn_probs(l))
    t1 = linear(o, W[p + "o.w"], W[p + "o.b"])
    z1 = x + t1 * masks.attn_out(l)
    h1, ln1 = layernorm(z1, W[p + "ln1.g"], W[p + "ln1.b"], cfg.ln_eps)
    u = linear(h1, W[p + "f1.w"], W[p + "f1.b"])
    g = gelu(u)
    t2 = linear(g, W[p + "f2.w"], W[p + "f2.b"])
    z2 = h1 + t2 * masks.ffn_out(l)
    y, ln2 = layernorm(z2, W[p + "ln2.g"], W[p + "ln2.b"], cfg.ln_eps)
    cache = dict(x=x, qkv=qkv, o=o, acache=acache, ln1=ln1, h1=h1, u=u, g=g, ln2=ln2)
    return y, cache


def layer_bwd(cfg, W, l, dy, c, B, S, masks: Masks, G):
    """post-LN layer backward."""
    p = f"layer{l}."
    dz2, G[p + "ln2.g"], G[p + "ln2.b"] = layernorm_bwd(dy, c["ln2"], W[p + "ln2.g"])
    dt2 = dz2 * masks.ffn_out(l)
    dg, G[p + "f2.w"], G[p + "f2.b"] = linear_bwd(dt2, c["g"], W[p + "f2.w"])
    du = gelu_bwd(dg, c["u"])
    dh1, G[p + "f1.w"], G[p + "f1.b"] = linear_bwd(du, c["h1"], W[p + "f1.w"])
    dh1 = dh1 + dz2
    dz1, G[p + "ln1.g"], G[p + "ln1.b"] = layernorm_bwd(dh1, c["ln1"], W[p + "ln1.g"])
    dt1 = dz1 * masks.attn_out(l)
    do, G[p + "o.w"], G[p + "o.b"] = linear_bwd(dt1, c["o"], W[p + "o.w"])
    dqkv = attention_bwd(do, c["acache"], B, S, cfg.heads, masks.attn_probs(l))
    dx, G[p + "qkv.w"], G[p + "qkv.b"] = linear_bwd(dqkv, c["x"], W[p + "qkv.w"])
    return dx + dz1


# --------------------------------------------------------------------------
# GPT-2 pre-LN layer (causal): a = LN1(x); r1 = x + drop(Attn(a) Wo + bo);
# m = LN2(r1); y = r1 + drop(gelu_tanh(m W1 + b1) W2 + b2)
# --------------------------------------------------------------------------

def layer_fwd_pre(cfg, W, l, x, lengths, B, S, masks: Masks, causal: bool = True):
    p = f"layer{l}."
    a, ln1 = layernorm(x, W[p + "ln1.g"], W[p + "ln1.b"], cfg.ln_eps)
    qkv = linear(a, W[p + "qkv.w"], W[p + "qkv.b"])
    o, acache = attention_fwd(qkv, lengths, B, S, cfg.heads, masks.attn_probs(l), causal=causal)
    r1 = x + linear(o, W[p + "o.w"], W[p + "o.b"]) * masks.attn_out(l)
    m, ln2 = layernorm(r1, W[p + "ln2.g"], W[p + "ln2.b"], cfg.ln_eps)
    u = linear(m, W[p + "f1.w"], W[p + "f1.b"])
    g = gelu_tanh(u)
    y = r1 + linear(g, W[p + "f2.w"], W[p + "f2.b"]) * masks.ffn_out(l)
    return y, dict(a=a, ln1=ln1, qkv=qkv, o=o, acache=acache, m=m, ln2=ln2, u=u, g=g)


def layer_bwd_pre(cfg, W, l, dy, c, B, S, masks: Masks, G):
    p = f"layer{l}."
    dt2 = dy * masks.ffn_out(l)
    dg, G[p + "f2.w"], G[p + "f2.b"] = linear_bwd(dt2, c["g"], W[p + "f2.w"])
    du = gelu_tanh_bwd(dg, c["u"])
    dm, G[p + "f1.w"], G[p + "f1.b"] = linear_bwd(du, c["m"], W[p + "f1.w"])
    dr1_ln, G[p + "ln2.g"], G[p + "ln2.b"] = layernorm_bwd(dm, c["ln2"], W[p + "ln2.g"])
    dr1 = dy + dr1_ln
    dt1 = dr1 * masks.attn_out(l)
    do, G[p + "o.w"], G[p + "o.b"] = linear_bwd(dt1, c["o"], W[p + "o.w"])
    dqkv = attention_bwd(do, c["acache"], B, S, cfg.heads, masks.attn_probs(l))
    da, G[p + "qkv.w"], G[p + "qkv.b"] = linear_bwd(dqkv, c["a"], W[p + "qkv.w"])
    dx_ln, G[p + "ln1.g"], G[p + "ln1.b"] = layernorm_bwd(da, c["ln1"], W[p + "ln1.g"])
    return dr1 + dx_ln


# --------------------------------------------------------------------------
# embeddings and heads
# --------------------------------------------------------------------------

def embed_fwd(cfg, W, batch: Batch, masks: Masks):
    if cfg.arch == ARCH_PRE_LN:                   # GPT-2: drop(wte[ids] + wpe[pos]), no LN
        B, S = batch.input_ids.shape
        ids = batch.input_ids.reshape(-1)
        pos = np.tile(np.arange(S) + cfg.pos_offset, B)
        return (W["emb.word"][ids] + W["emb.pos"][pos]) * masks.emb(), (ids, pos, None, None)
    B, S = batch.input_ids.shape
    ids = batch.input_ids.reshape(-1)
    pos = np.tile(np.arange(S) + cfg.pos_offset, B)
    tt = batch.token_type.reshape(-1)
    z0 = W["emb.word"][ids] + W["emb.pos"][pos] + W["emb.type"][tt]
    ln0, cache = layernorm(z0, W["emb.ln.g"], W["emb.ln.b"], cfg.ln_eps)
    return ln0 * masks.emb(), (ids, pos, tt, cache)


def embed_bwd(cfg, W, dx1, ec, masks: Masks, G):
    ids, pos, tt, cache = ec
    if cfg.arch == ARCH_PRE_LN:                   # tied wte: add to the LM-head gradient
        dz0 = dx1 * masks.emb()
        np.add.at(G["emb.word"], ids, dz0)
        acc = np.zeros_like(W["emb.pos"])
        np.add.at(acc, pos, dz0)
        G["emb.pos"] = acc
        return
    dln0 = dx1 * masks.emb()
    dz0, G["emb.ln.g"], G["emb.ln.b"] = layernorm_bwd(dln0, cache, W["emb.ln.g"])
    for name, idx in (("emb.word", ids), ("emb.pos", pos), ("emb.type", tt)):
        acc = np.zeros_like(W[name])
        np.add.at(acc, idx, dz0)
        G[name] = acc
    # HF padding_idx semantics (reading A24, BERT/RoBERTa): the pad token's
    # embedding row gets no gradient.  (Its accumulated value is 0 anyway: padded
    # rows carry zero gradient because no loss term reads them, A26.)
    G["emb.word"][cfg.pad_id] = 0.0


def head_fwd_bwd(cfg, W, y, batch: Batch, masks: Masks, G):
    """Loss and dL/dy for the task head; fills head grads into G."""
    B, S = batch.input_ids.shape
    H = cfg.hidden
    dy = np.zeros_like(y)
    if cfg.head in (HEAD_SEQCLS, HEAD_MC):
        rows = np.arange(B) * S                        # CLS token of every sequence
        c = y[rows]
        pl = np.tanh(linear(c, W["pool.w"], W["pool.b"]))
        pd = pl * masks.head()
        logits = linear(pd, W["cls.w"], W["cls.b"])    # [B, n_out]
        if cfg.head == HEAD_MC:
            logits2 = logits.reshape(B // cfg.n_choices, cfg.n_choices)
            loss, dl2 = ce_rows(logits2, batch.labels)
            dlogits = dl2.reshape(B, 1)
        else:
            loss, dlogits = ce_rows(logits, batch.labels)
        dpd, G["cls.w"], G["cls.b"] = linear_bwd(dlogits, pd, W["cls.w"])
        dpre = dpd * masks.head() * (1.0 - pl * pl)
        dc, G["pool.w"], G["pool.b"] = linear_bwd(dpre, c, W["pool.w"])
        dy[rows] = dc
        return loss, dy
    if cfg.head == HEAD_LM:
        # final LN -> tied vocabulary projection -> next-token CE over s < len-1 (pads ignored)
        hf, lnf = layernorm(y, W["lnf.g"], W["lnf.b"], cfg.ln_eps)
        logits = hf @ W["emb.word"].T                                   # [T, V]
        ids = batch.input_ids
        valid = np.zeros((B, S), bool)
        tgt = np.zeros((B, S), np.int64)
        for b in range(B):
            n = int(batch.lengths[b])
            valid[b, :max(n - 1, 0)] = True
            tgt[b, :max(n - 1, 0)] = ids[b, 1:n]
        rows = np.nonzero(valid.reshape(-1))[0]
        loss, dl = ce_rows(logits[rows], tgt.reshape(-1)[rows])
        dlog = np.zeros_like(logits)
        dlog[rows] = dl
        dhf = dlog @ W["emb.word"]
        G["emb.word"] = dlog.T @ hf
        dy, G["lnf.g"], G["lnf.b"] = layernorm_bwd(dhf, lnf, W["lnf.g"])
        return loss, dy
    # QA span head: start/end logits over valid positions (pads masked, R-A26)
    logits = linear(y, W["qa.w"], W["qa.b"]).reshape(B, S, 2)
    valid = np.arange(S)[None, :] < batch.lengths[:, None]
    dlog = np.zeros_like(logits)
    loss = 0.0
    for j in range(2):
        lg = np.where(valid, logits[:, :, j], -np.inf)
        lj, dj = ce_rows(lg, batch.labels[j::2])
        loss += 0.5 * lj
        dlog[:, :, j] = 0.5 * np.where(valid, dj, 0.0)
    dlog = dlog.reshape(B * S, 2)
    dy, G["qa.w"], G["qa.b"] = linear_bwd(dlog, y, W["qa.w"])
    return loss, dy


# --------------------------------------------------------------------------
# the whole step
# --------------------------------------------------------------------------

def train_step_grads(cfg: ModelConfig, params: Dict[str, np.ndarray], batch: Batch,
                     seed: int, step: int, rank: int = 0,
                     plan: Optional[Sequence[int]] = None, p: Optional[float] = None,
                     mask_override=None):
    """Loss and fp64 gradients of one mini-batch.

    ``plan`` = 0-based indices of dropped layers: their caches are discarded
    after forward (only the layer input is kept) and re-created by replaying
    the forward right before their backward."""
    if cfg.arch == ARCH_ENCDEC:
        return encdec_step_grads(cfg, params, batch, seed, step, rank, plan, p)
    W = {k: np.asarray(v, np.float64) for k, v in params.items()}
    B, S = batch.input_ids.shape
    masks = Masks(cfg, B, S, seed, step, rank, p, mask_override)
    dropped = set(plan or ())
    G: Dict[str, np.ndarray] = {}
    x, ec = embed_fwd(cfg, W, batch, masks)
    caches, inputs = [], []
    fwd = layer_fwd_pre if cfg.arch == ARCH_PRE_LN else layer_fwd
    bwd = layer_bwd_pre if cfg.arch == ARCH_PRE_LN else layer_bwd
    for l in range(cfg.n_layers):
        inputs.append(x)
        x, c = fwd(cfg, W, l, x, batch.lengths, B, S, masks)
        caches.append(None if l in dropped else c)
    loss, dy = head_fwd_bwd(cfg, W, x, batch, masks, G)
    for l in reversed(range(cfg.n_layers)):
        c = caches[l]
        if c is None:                                   # recompute (replay)
            _, c = fwd(cfg, W, l, inputs[l], batch.lengths, B, S, masks)
        dy = bwd(cfg, W, l, dy, c, B, S, masks, G)
        caches[l] = None
    embed_bwd(cfg, W, dy, ec, masks, G)
    return loss, G


# --------------------------------------------------------------------------
# encoder-decoder (Table II TR-T5; reading A32): pre-LN
# encoder layers (bidirectional) + the encoder's final LN -> enc_out; pre-LN
# decoder layers: r1 = x + drop(SelfAttn_causal(LN1 x)); r2 = r1 +
# drop(CrossAttn(LN2 r1, enc_out)); y = r2 + drop(FFN(LN3 r2)); the decoder's
# final LN -> tied LM head, next-token CE over the target.  Dropout sites
# (R-B): encoder layers l = 0..Le-1, decoder layers Le + j; the decoder
# embedding uses layer field DEC_EMB; cross-attention kinds 5 (probabilities,
# element ((b h + head) S_t + q) S_s + k) and 6 (output hidden).
# --------------------------------------------------------------------------

DEC_EMB = 0xFFE
KIND_CROSS_PROBS = 5
KIND_CROSS_OUT = 6


class EncDecMasks:
    def __init__(self, cfg, B, Ss, St, seed, step, rank=0, p=None):
        self.cfg, self.B, self.Ss, self.St = cfg, B, Ss, St
        self.seed, self.step, self.rank = seed, step, rank
        self.p = cfg.p_drop if p is None else p
        self.enc = Masks(cfg, B, Ss, seed, step, rank, p)          # encoder layers, encoder embedding
        self.dec = Masks(cfg, B, St, seed, step, rank, p)          # decoder self-attn / hidden sites

    def _m(self, n, kind, layer, shape):
        if self.p <= 0.0:
            return np.ones(shape)
        keep = px.keep_mask(n, self.p, self.seed, px.site_word(kind, layer, self.rank), self.step)
        return keep.reshape(shape).astype(np.float64) / (1.0 - self.p)

    def dec_emb(self):
        T, H = self.B * self.St, self.cfg.hidden
        return self._m(T * H, px.KIND_EMB, DEC_EMB, (T, H))

    def cross_probs(self, layer):
        B, h = self.B, self.cfg.heads
        return self._m(B * h * self.St * self.Ss, KIND_CROSS_PROBS, layer, (B, h, self.St, self.Ss))

    def cross_out(self, layer):
        T, H = self.B * self.St, self.cfg.hidden
        return self._m(T * H, KIND_CROSS_OUT, layer, (T, H))


def cross_attention_fwd(q, kv, klen, B, St, Ss, h, pmask):
    """O = drop(softmax(Q K^T / sqrt d + key-pad mask)) V with queries from the
    decoder [B*St, H] and keys / values from the encoder [B*Ss, 2H]."""
    H = q.shape[1]
    d = H // h
    qh = q.reshape(B, St, h, d).transpose(0, 2, 1, 3)
    k = kv[:, :H].reshape(B, Ss, h, d).transpose(0, 2, 1, 3)
    v = kv[:, H:].reshape(B, Ss, h, d).transpose(0, 2, 1, 3)
    s = qh @ k.transpose(0, 1, 3, 2) / math.sqrt(d)
    keyvalid = np.arange(Ss)[None, :] < np.asarray(klen)[:, None]
    s = np.where(np.broadcast_to(keyvalid[:, None, None, :], s.shape), s, -np.inf)
    p, lse = softmax_lastdim(s)
    pd = p * pmask
    o = (pd @ v).transpose(0, 2, 1, 3).reshape(B * St, H)
    return o, (qh, k, v, p, pd)


def cross_attention_bwd(dout, cache, B, St, Ss, h, pmask):
    """-> dQ [B*St, H], dKV [B*Ss, 2H]."""
    qh, k, v, p, pd = cache
    d = qh.shape[-1]
    H = h * d
    do = dout.reshape(B, St, h, d).transpose(0, 2, 1, 3)
    dv = pd.transpose(0, 1, 3, 2) @ do
    dp = (do @ v.transpose(0, 1, 3, 2)) * pmask
    ds = p * (dp - (dp * p).sum(axis=-1, keepdims=True))
    dq = ds @ k / math.sqrt(d)
    dk = ds.transpose(0, 1, 3, 2) @ qh / math.sqrt(d)
    flat = lambda t, S: t.transpose(0, 2, 1, 3).reshape(B * S, H)
    return flat(dq, St), np.concatenate([flat(dk, Ss), flat(dv, Ss)], axis=1)


def dec_layer_fwd(cfg, W, j, x, enc_out, tlen, slen, B, St, Ss, mk: EncDecMasks):
    p, L = f"dec{j}.", cfg.n_layers + j                      # dropout layer field
    a, ln1 = layernorm(x, W[p + "ln1.g"], W[p + "ln1.b"], cfg.ln_eps)
    qkv = linear(a, W[p + "qkv.w"], W[p + "qkv.b"])
    o, ac = attention_fwd(qkv, tlen, B, St, cfg.heads, mk.dec.attn_probs(L), causal=True)
    r1 = x + linear(o, W[p + "o.w"], W[p + "o.b"]) * mk.dec.attn_out(L)
    c, ln2 = layernorm(r1, W[p + "ln2.g"], W[p + "ln2.b"], cfg.ln_eps)
    qc = linear(c, W[p + "cq.w"], W[p + "cq.b"])
    kvc = linear(enc_out, W[p + "ckv.w"], W[p + "ckv.b"])
    oc, cc = cross_attention_fwd(qc, kvc, slen, B, St, Ss, cfg.heads, mk.cross_probs(L))
    r2 = r1 + linear(oc, W[p + "co.w"], W[p + "co.b"]) * mk.cross_out(L)
    m, ln3 = layernorm(r2, W[p + "ln3.g"], W[p + "ln3.b"], cfg.ln_eps)
    u = linear(m, W[p + "f1.w"], W[p + "f1.b"])
    g = gelu_tanh(u)
    y = r2 + linear(g, W[p + "f2.w"], W[p + "f2.b"]) * mk.dec.ffn_out(L)
    return y, dict(a=a, ln1=ln1, qkv=qkv, o=o, ac=ac, c=c, ln2=ln2, qc=qc, oc=oc, cc=cc, m=m, ln3=ln3, u=u, g=g)


def dec_layer_bwd(cfg, W, j, dy, cch, enc_out, B, St, Ss, mk: EncDecMasks, G):
    """-> (dx, d enc_out contribution)."""
    p, L = f"dec{j}.", cfg.n_layers + j
    dt3 = dy * mk.dec.ffn_out(L)
    dg, G[p + "f2.w"], G[p + "f2.b"] = linear_bwd(dt3, cch["g"], W[p + "f2.w"])
    du = gelu_tanh_bwd(dg, cch["u"])
    dm, G[p + "f1.w"], G[p + "f1.b"] = linear_bwd(du, cch["m"], W[p + "f1.w"])
    dr2_ln, G[p + "ln3.g"], G[p + "ln3.b"] = layernorm_bwd(dm, cch["ln3"], W[p + "ln3.g"])
    dr2 = dy + dr2_ln
    dtc = dr2 * mk.cross_out(L)
    doc, G[p + "co.w"], G[p + "co.b"] = linear_bwd(dtc, cch["oc"], W[p + "co.w"])
    dqc, dkvc = cross_attention_bwd(doc, cch["cc"], B, St, Ss, cfg.heads, mk.cross_probs(L))
    dc, G[p + "cq.w"], G[p + "cq.b"] = linear_bwd(dqc, cch["c"], W[p + "cq.w"])
    denc, G[p + "ckv.w"], G[p + "ckv.b"] = linear_bwd(dkvc, enc_out, W[p + "ckv.w"])
    dr1_ln, G[p + "ln2.g"], G[p + "ln2.b"] = layernorm_bwd(dc, cch["ln2"], W[p + "ln2.g"])
    dr1 = dr2 + dr1_ln
    dt1 = dr1 * mk.dec.attn_out(L)
    do, G[p + "o.w"], G[p + "o.b"] = linear_bwd(dt1, cch["o"], W[p + "o.w"])
    dqkv = attention_bwd(do, cch["ac"], B, St, cfg.heads, mk.dec.attn_probs(L))
    da, G[p + "qkv.w"], G[p + "qkv.b"] = linear_bwd(dqkv, cch["a"], W[p + "qkv.w"])
    dx_ln, G[p + "ln1.g"], G[p + "ln1.b"] = layernorm_bwd(da, cch["ln1"], W[p + "ln1.g"])
    return dr1 + dx_ln, denc


def encdec_step_grads(cfg: ModelConfig, params, batch: Batch, seed: int, step: int, rank: int = 0,
                      plan: Optional[Sequence[int]] = None, p: Optional[float] = None):
    """Loss and fp64 gradients of one encoder-decoder step; ``plan`` = dropped
    layers over the Le + Ld units (encoder l, decoder Le + j): discarded
    caches replayed before their backward (c-C identity)."""
    W = {k: np.asarray(v, np.float64) for k, v in params.items()}
    B, Ss = batch.input_ids.shape
    St = batch.dec_len
    Le, Ld = cfg.n_layers, cfg.n_dec_layers
    mk = EncDecMasks(cfg, B, Ss, St, seed, step, rank, p)
    dropped = set(plan or ())
    G: Dict[str, np.ndarray] = {}
    # encoder
    ids = batch.input_ids.reshape(-1)
    pos = np.tile(np.arange(Ss) + cfg.pos_offset, B)
    x = (W["emb.word"][ids] + W["emb.pos"][pos]) * mk.enc.emb()
    enc_in, enc_c = [], []
    for l in range(Le):
        enc_in.append(x)
        x, c = layer_fwd_pre(cfg, W, l, x, batch.lengths, B, Ss, mk.enc, causal=False)
        enc_c.append(None if l in dropped else c)
    enc_out, lne = layernorm(x, W["enc.lnf.g"], W["enc.lnf.b"], cfg.ln_eps)
    # decoder
    tids = batch.dec_ids.reshape(-1)
    tpos = np.tile(np.arange(St) + cfg.pos_offset, B)
    xd = (W["emb.word"][tids] + W["emb.pos"][tpos]) * mk.dec_emb()
    dec_in, dec_c = [], []
    for j in range(Ld):
        dec_in.append(xd)
        xd, c = dec_layer_fwd(cfg, W, j, xd, enc_out, batch.dec_lengths, batch.lengths, B, St, Ss, mk)
        dec_c.append(None if Le + j in dropped else c)
    # LM head on the decoder (final LN, tied vocabulary projection, next-token CE)
    tb = Batch(batch.dec_ids, np.zeros_like(batch.dec_ids), batch.dec_lengths, np.zeros(0, np.int32), St)
    loss, dy = head_fwd_bwd(cfg, W, xd, tb, mk.dec, G)
    denc = np.zeros_like(enc_out)
    for j in reversed(range(Ld)):
        c = dec_c[j]
        if c is None:
            _, c = dec_layer_fwd(cfg, W, j, dec_in[j], enc_out, batch.dec_lengths, batch.lengths, B, St, Ss, mk)
        dy, de = dec_layer_bwd(cfg, W, j, dy, c, enc_out, B, St, Ss, mk, G)
        denc += de
    # decoder embedding (tied wte: the LM head's dW_e is in G["emb.word"])
    dz = dy * mk.dec_emb()
    np.add.at(G["emb.word"], tids, dz)
    dpos = np.zeros_like(W["emb.pos"])
    np.add.at(dpos, tpos, dz)
    # encoder
    dx, G["enc.lnf.g"], G["enc.lnf.b"] = layernorm_bwd(denc, lne, W["enc.lnf.g"])
    for l in reversed(range(Le)):
        c = enc_c[l]
        if c is None:
            _, c = layer_fwd_pre(cfg, W, l, enc_in[l], batch.lengths, B, Ss, mk.enc, causal=False)
        dx = layer_bwd_pre(cfg, W, l, dx, c, B, Ss, mk.enc, G)
    dz = dx * mk.enc.emb()
    np.add.at(G["emb.word"], ids, dz)
    np.add.at(dpos, pos, dz)
    G["emb.pos"] = dpos
    return loss, G


def adamw(params, grads, m, v, t, lr, beta1=0.9, beta2=0.999, eps=1e-8, wd=0.0):
    """torch.optim.AdamW semantics (R-A25), fp64, applied to every tensor.
    Returns new (params, m, v); t is the 1-based step count."""
    out_p, out_m, out_v = {}, {}, {}
    bc1 = 1.0 - beta1 ** t
    bc2 = 1.0 - beta2 ** t
    for k in params:
        pk = np.asarray(params[k], np.float64) * (1.0 - lr * wd)
        mk = beta1 * m[k] + (1.0 - beta1) * grads[k]
        vk = beta2 * v[k] + (1.0 - beta2) * grads[k] * grads[k]
        denom = np.sqrt(vk) / math.sqrt(bc2) + eps
        out_p[k] = pk - (lr / bc1) * mk / denom
        out_m[k], out_v[k] = mk, vk
    return out_p, out_m, out_v
