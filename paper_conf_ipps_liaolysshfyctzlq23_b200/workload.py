"""Seeded synthetic workloads: model configs, parameter spec, weights and batches.

This module is the ONLY code shared by the product path (binding, bench) and
the test oracle (``oracle/``).  It holds no arithmetic of the method: it only
draws seeded random numbers with the shapes, sizes and length mixes of the
paper's workloads.

Workload shapes follow PAPER.md:
  * P:73 (§III-A) input size = numel of the mini-batch input, ranges such as
    SWAG 35~141, SQuAD 153~512 tokens; P:49 (§II-A) samples of a mini-batch are
    padded to the longest sample.
  * Table II tasks / batch sizes: MC-Roberta bs 16 (x4 choices),
    QA-Bert bs 12.
"""
from __future__ import annotations

import dataclasses
import math
from typing import Dict, List, Optional, Tuple

import numpy as np

ARCH_POST_LN = 0     # BERT / RoBERTa post-LN encoder
ARCH_PRE_LN = 1      # GPT-2 pre-LN causal decoder stack
ARCH_ENCDEC = 2      # T5-like encoder-decoder: pre-LN encoder + pre-LN decoder with cross-attention
HEAD_SEQCLS = 0      # pooler -> dropout -> linear(n_labels) -> CE
HEAD_MC = 1          # pooler -> dropout -> linear(1) -> [B_q, n_choices] -> CE
HEAD_QA = 2          # linear(2) on every token -> start/end CE
HEAD_LM = 3          # final LN -> tied vocabulary projection -> next-token CE


@dataclasses.dataclass(frozen=True)
class ModelConfig:
    name: str
    cfg_id: int
    n_layers: int
    hidden: int
    heads: int
    ffn: int
    vocab: int
    max_pos: int
    type_vocab: int
    pos_offset: int
    head: int
    n_choices: int          # MC only (sequences per question)
    n_labels: int           # seq-cls only
    dtype: str              # "fp32" | "bf16"
    ln_eps: float
    p_drop: float
    # workload
    n_seqs: int             # sequences per GPU per step (B_seq)
    seq_lo: int
    seq_hi: int
    pad: int                # S_pad is rounded up to a multiple of this
    budget_frac: float
    cls_id: int
    sep_id: int
    pad_id: int
    first_tok: int
    arch: int = ARCH_POST_LN
    # heterogeneous stages: FFN width of every layer; () = ffn everywhere
    ffn_layers: Tuple[int, ...] = ()
    # encoder-decoder: decoder layers (n_layers = encoder layers)
    n_dec_layers: int = 0

    def ffn_of(self, l: int) -> int:
        return self.ffn_layers[l] if self.ffn_layers else self.ffn

    @property
    def causal(self) -> bool:
        return self.arch == ARCH_PRE_LN

    @property
    def n_units_total(self) -> int:
        """Checkpointable layers: encoder + decoder layers for ARCH_ENCDEC."""
        return self.n_layers + self.n_dec_layers

    @property
    def head_dim(self) -> int:
        return self.hidden // self.heads

    @property
    def n_out(self) -> int:
        if self.head == HEAD_SEQCLS:
            return self.n_labels
        if self.head == HEAD_MC:
            return 1
        if self.head == HEAD_LM:
            return self.vocab
        return 2

    @property
    def samples_per_step(self) -> int:
        """Training examples per GPU per step (MC: questions, else sequences)."""
        if self.head == HEAD_MC:
            return self.n_seqs // self.n_choices
        return self.n_seqs

    @property
    def n_label_values(self) -> int:
        """int32 label values per step (documented in include/mimose.h)."""
        if self.head == HEAD_MC:
            return self.n_seqs // self.n_choices
        if self.head == HEAD_QA:
            return 2 * self.n_seqs
        if self.head == HEAD_LM:
            return 0                      # targets are the next input tokens
        return self.n_seqs

    @property
    def max_seq(self) -> int:
        return ((self.seq_hi + self.pad - 1) // self.pad) * self.pad


CONFIGS: Dict[str, ModelConfig] = {
    # BASELINE.json configs[0]: toy 2-layer encoder hidden=64 heads=2, batch=2,
    # seq len uniform in [8,32], fp32, budget 50% of the no-checkpoint peak.
    "toy": ModelConfig("toy", 0, 2, 64, 2, 256, 1000, 32, 2, 0, HEAD_SEQCLS, 1, 2,
                       "fp32", 1e-12, 0.1, 2, 8, 32, 1, 0.5, 101, 102, 0, 103),
    # configs[1]: BERT-base, SWAG-like multiple choice, 16 q x 4 choices, 32-128.
    "bert-base": ModelConfig("bert-base", 1, 12, 768, 12, 3072, 30522, 512, 2, 0,
                             HEAD_MC, 4, 2, "bf16", 1e-12, 0.1, 64, 32, 128, 8, 0.6,
                             101, 102, 0, 103),
    # configs[2]: BERT-large, SQuAD-like QA, seq 128-512, batch 12 (Table II QA-Bert).
    "bert-large": ModelConfig("bert-large", 2, 24, 1024, 16, 4096, 30522, 512, 2, 0,
                              HEAD_QA, 1, 2, "bf16", 1e-12, 0.1, 12, 128, 512, 8, 0.5,
                              101, 102, 0, 103),
    # configs[3]: RoBERTa-large, MC (Table II MC-Roberta), seq 64-512.
    "roberta-large": ModelConfig("roberta-large", 3, 24, 1024, 16, 4096, 50265, 514, 1, 2,
                                 HEAD_MC, 4, 2, "bf16", 1e-5, 0.1, 64, 64, 512, 8, 0.5,
                                 0, 2, 1, 3),
    # configs[4]: GPT-2 medium, causal pre-LN, seq 256-1024, budget 40%, 8 sequences
    # per GPU (batch not given in BASELINE; chosen).  No special tokens but the
    # end-of-text id 50256, used as the pad id.
    "gpt2-medium": ModelConfig("gpt2-medium", 4, 24, 1024, 16, 4096, 50257, 1024, 0, 0,
                               HEAD_LM, 1, 2, "bf16", 1e-5, 0.1, 8, 256, 1024, 8, 0.4,
                               50256, 50256, 50256, 0, ARCH_PRE_LN),
    # heterogeneous stages.  A synthetic BERT-base-width
    # encoder whose three 4-layer stages differ in FFN width (4096 / 3072 / 1536),
    # so the per-layer activation size falls stage by stage (1.15 : 1 : 0.78 per
    # token) as in Swin or ResNet, whose first stage holds the largest
    # activations (Fig. 9); SWAG-like MC batches, the BERT-base
    # length schedule, budget 60%.
    "hetero": ModelConfig("hetero", 5, 12, 768, 12, 4096, 30522, 512, 2, 0,
                          HEAD_MC, 4, 2, "bf16", 1e-12, 0.1, 64, 32, 128, 8, 0.6,
                          101, 102, 0, 103, ARCH_POST_LN, (4096,) * 4 + (3072,) * 4 + (1536,) * 4),
    # the paper's TR-T5 task (Table II: T5-base on UN_PC, batch 8;
    # P:73 input sizes 17-460).  T5-base shapes (12 + 12 layers, H 768, 12 heads,
    # F 3072, 32128-word tied vocabulary) with pre-LN blocks (T5 is pre-norm),
    # biases and tanh-GELU kept, absolute positions (reading A32); source
    # lengths 17-460, target = source x U[0.8, 1.2]; budget 50%.
    "t5-base": ModelConfig("t5-base", 6, 12, 768, 12, 3072, 32128, 512, 0, 0,
                           HEAD_LM, 1, 2, "bf16", 1e-6, 0.1, 8, 17, 460, 8, 0.5,
                           1, 1, 0, 3, ARCH_ENCDEC, (), 12),
}


def small_config(base: str, **over) -> ModelConfig:
    """A reduced-width/depth variant used by parity tests (same structure)."""
    return dataclasses.replace(CONFIGS[base], **over)


# ---------------------------------------------------------------------------
# Parameter spec: the documented flat order of include/mimose.h
# ---------------------------------------------------------------------------

def param_spec(cfg: ModelConfig) -> List[Tuple[str, Tuple[int, ...]]]:
    H, F, V = cfg.hidden, cfg.ffn, cfg.vocab
    P = cfg.max_pos
    if cfg.arch == ARCH_ENCDEC:
        # shared wte (encoder input, decoder input, tied LM head), wpe; pre-LN
        # encoder layers, the encoder's final LN; pre-LN decoder layers with a
        # cross-attention block (LN2 -> Q from the decoder, K/V from the encoder
        # output); the decoder's final LN
        spec = [("emb.word", (V, H)), ("emb.pos", (P, H))]
        for l in range(cfg.n_layers):
            p = f"layer{l}."
            spec += [(p + "ln1.g", (H,)), (p + "ln1.b", (H,)), (p + "qkv.w", (3 * H, H)), (p + "qkv.b", (3 * H,)),
                     (p + "o.w", (H, H)), (p + "o.b", (H,)), (p + "ln2.g", (H,)), (p + "ln2.b", (H,)),
                     (p + "f1.w", (F, H)), (p + "f1.b", (F,)), (p + "f2.w", (H, F)), (p + "f2.b", (H,))]
        spec += [("enc.lnf.g", (H,)), ("enc.lnf.b", (H,))]
        for j in range(cfg.n_dec_layers):
            p = f"dec{j}."
            spec += [(p + "ln1.g", (H,)), (p + "ln1.b", (H,)), (p + "qkv.w", (3 * H, H)), (p + "qkv.b", (3 * H,)),
                     (p + "o.w", (H, H)), (p + "o.b", (H,)),
                     (p + "ln2.g", (H,)), (p + "ln2.b", (H,)), (p + "cq.w", (H, H)), (p + "cq.b", (H,)),
                     (p + "ckv.w", (2 * H, H)), (p + "ckv.b", (2 * H,)), (p + "co.w", (H, H)), (p + "co.b", (H,)),
                     (p + "ln3.g", (H,)), (p + "ln3.b", (H,)),
                     (p + "f1.w", (F, H)), (p + "f1.b", (F,)), (p + "f2.w", (H, F)), (p + "f2.b", (H,))]
        spec += [("lnf.g", (H,)), ("lnf.b", (H,))]
        return spec
    if cfg.arch == ARCH_PRE_LN:
        # GPT-2: wte (tied with the LM head), wpe; pre-LN layers; final LN
        spec = [("emb.word", (V, H)), ("emb.pos", (P, H))]
        for l in range(cfg.n_layers):
            p = f"layer{l}."
            F = cfg.ffn_of(l)
            spec += [
                (p + "ln1.g", (H,)), (p + "ln1.b", (H,)),
                (p + "qkv.w", (3 * H, H)), (p + "qkv.b", (3 * H,)),
                (p + "o.w", (H, H)), (p + "o.b", (H,)),
                (p + "ln2.g", (H,)), (p + "ln2.b", (H,)),
                (p + "f1.w", (F, H)), (p + "f1.b", (F,)),
                (p + "f2.w", (H, F)), (p + "f2.b", (H,)),
            ]
        spec += [("lnf.g", (H,)), ("lnf.b", (H,))]
        return spec
    spec: List[Tuple[str, Tuple[int, ...]]] = [
        ("emb.word", (V, H)), ("emb.pos", (P, H)), ("emb.type", (cfg.type_vocab, H)),
        ("emb.ln.g", (H,)), ("emb.ln.b", (H,)),
    ]
    for l in range(cfg.n_layers):
        p = f"layer{l}."
        F = cfg.ffn_of(l)
        spec += [
            (p + "qkv.w", (3 * H, H)), (p + "qkv.b", (3 * H,)),
            (p + "o.w", (H, H)), (p + "o.b", (H,)),
            (p + "ln1.g", (H,)), (p + "ln1.b", (H,)),
            (p + "f1.w", (F, H)), (p + "f1.b", (F,)),
            (p + "f2.w", (H, F)), (p + "f2.b", (H,)),
            (p + "ln2.g", (H,)), (p + "ln2.b", (H,)),
        ]
    if cfg.head in (HEAD_SEQCLS, HEAD_MC):
        spec += [("pool.w", (H, H)), ("pool.b", (H,)),
                 ("cls.w", (cfg.n_out, H)), ("cls.b", (cfg.n_out,))]
    else:
        spec += [("qa.w", (2, H)), ("qa.b", (2,))]
    return spec


def n_params(cfg: ModelConfig) -> int:
    return sum(int(np.prod(s)) for _, s in param_spec(cfg))


def init_params(cfg: ModelConfig, parity: bool = False, seed: int | None = None) -> Dict[str, np.ndarray]:
    """Seeded weights (fp32).  BERT init N(0, 0.02^2); with ``parity`` the biases,
    LN gains and shifts are random too so every gradient path is exercised."""
    rng = np.random.Generator(np.random.PCG64(1000 + cfg.cfg_id if seed is None else seed))
    out: Dict[str, np.ndarray] = {}
    for name, shape in param_spec(cfg):
        leaf = name.rsplit(".", 1)[-1]
        if leaf == "g":
            v = rng.uniform(0.5, 1.5, shape) if parity else np.ones(shape)
        elif leaf == "b" and name.split(".")[-2].startswith("ln"):
            v = rng.normal(0.0, 0.1, shape) if parity else np.zeros(shape)
        elif leaf == "b":
            v = rng.normal(0.0, 0.02, shape) if parity else np.zeros(shape)
        else:
            v = rng.normal(0.0, 0.02, shape)
        out[name] = v.astype(np.float32)
    return out


def pack_params(cfg: ModelConfig, params: Dict[str, np.ndarray]) -> np.ndarray:
    """Concatenate in the documented order (no padding) -> fp32 host blob."""
    return np.concatenate([params[n].astype(np.float32).ravel() for n, _ in param_spec(cfg)])


def unpack_params(cfg: ModelConfig, blob: np.ndarray) -> Dict[str, np.ndarray]:
    out, off = {}, 0
    for name, shape in param_spec(cfg):
        n = int(np.prod(shape))
        out[name] = np.asarray(blob[off:off + n]).reshape(shape)
        off += n
    assert off == blob.size, (off, blob.size)
    return out


# ---------------------------------------------------------------------------
# Batches
# ---------------------------------------------------------------------------

@dataclasses.dataclass
class Batch:
    input_ids: np.ndarray    # int32 [B, S_pad]
    token_type: np.ndarray   # int32 [B, S_pad]
    lengths: np.ndarray      # int32 [B]
    labels: np.ndarray       # int32 [n_label_values]
    seq_len: int             # S_pad
    # encoder-decoder (ARCH_ENCDEC): the decoder's input ids, lengths, padded length
    dec_ids: Optional[np.ndarray] = None       # int32 [B, S_t_pad]
    dec_lengths: Optional[np.ndarray] = None   # int32 [B]
    dec_len: int = 0

    @property
    def input_size2(self) -> Tuple[int, int]:
        """The 2-D input size (source, target) of an encoder-decoder batch."""
        return int(self.input_ids.size), int(self.dec_ids.size) if self.dec_ids is not None else 0

    @property
    def n_seqs(self) -> int:
        return int(self.input_ids.shape[0])

    @property
    def input_size(self) -> int:
        """x of PAPER.md P:73: numel of the mini-batch input tensor."""
        return int(self.input_ids.size)


def roundup(v: int, m: int) -> int:
    return ((v + m - 1) // m) * m


def length_schedule(cfg: ModelConfig, n_steps: int, seed: int | None = None,
                    kind: str = "uniform") -> List[int]:
    """Longest-sequence length per step (shared by every DP rank).

    ``uniform``: U{lo..hi}.  ``normal``: truncated normal mu=(lo+hi)/2,
    sigma=(hi-lo)/4 ("normal distribution")."""
    rng = np.random.Generator(np.random.PCG64(2000 + cfg.cfg_id if seed is None else seed))
    out = []
    for _ in range(n_steps):
        if kind == "uniform":
            L = int(rng.integers(cfg.seq_lo, cfg.seq_hi + 1))
        else:
            mu, sd = (cfg.seq_lo + cfg.seq_hi) / 2, (cfg.seq_hi - cfg.seq_lo) / 4
            while True:
                L = int(round(rng.normal(mu, sd)))
                if cfg.seq_lo <= L <= cfg.seq_hi:
                    break
        out.append(L)
    return out


def make_batch(cfg: ModelConfig, longest: int, seed: int, n_seqs: int | None = None) -> Batch:
    """One synthetic mini-batch whose longest sequence has ``longest`` tokens,
    padded to S_pad = roundup(longest, cfg.pad)."""
    B = cfg.n_seqs if n_seqs is None else n_seqs
    rng = np.random.Generator(np.random.PCG64(seed))
    S = roundup(longest, cfg.pad)
    lens = np.empty(B, np.int32)
    lens[0] = longest
    lo = max(2, (longest + 1) // 2)
    if B > 1:
        lens[1:] = rng.integers(lo, longest + 1, size=B - 1)
    ids = np.full((B, S), cfg.pad_id, np.int32)
    tt = np.zeros((B, S), np.int32)
    for b in range(B):
        n = int(lens[b])
        if cfg.arch in (ARCH_PRE_LN, ARCH_ENCDEC):   # GPT-2 / T5 source: plain text tokens
            ids[b, :n] = rng.integers(cfg.first_tok, cfg.vocab - 1, size=n)
            continue
        ids[b, :n] = rng.integers(cfg.first_tok, cfg.vocab, size=n)
        ids[b, 0] = cfg.cls_id
        ids[b, n - 1] = cfg.sep_id
        if cfg.type_vocab > 1:
            tt[b, n // 2:n] = 1
    if cfg.arch == ARCH_ENCDEC:
        # target: longest = source longest x U[0.8, 1.2] within [seq_lo/2, seq_hi]
        # (translation pairs of similar length, UN_PC-like); next-token CE on it
        Lt = int(np.clip(round(longest * rng.uniform(0.8, 1.2)), max(2, cfg.seq_lo // 2), cfg.seq_hi))
        St = roundup(Lt, cfg.pad)
        tl = np.empty(B, np.int32)
        tl[0] = Lt
        if B > 1:
            tl[1:] = rng.integers(max(2, (Lt + 1) // 2), Lt + 1, size=B - 1)
        did = np.full((B, St), cfg.pad_id, np.int32)
        for b in range(B):
            did[b, :int(tl[b])] = rng.integers(cfg.first_tok, cfg.vocab, size=int(tl[b]))
        return Batch(ids, tt, lens, np.zeros(0, np.int32), S, did, tl, St)
    if cfg.head == HEAD_LM:
        labels = np.zeros(0, np.int32)
    elif cfg.head == HEAD_SEQCLS:
        labels = rng.integers(0, cfg.n_labels, size=B).astype(np.int32)
    elif cfg.head == HEAD_MC:
        labels = rng.integers(0, cfg.n_choices, size=B // cfg.n_choices).astype(np.int32)
    else:
        labels = np.empty(2 * B, np.int32)
        for b in range(B):
            n = int(lens[b])
            s0 = int(rng.integers(1, max(2, n - 1)))
            e0 = int(rng.integers(s0, min(s0 + 30, max(s0 + 1, n - 1))))
            labels[2 * b], labels[2 * b + 1] = s0, min(e0, n - 1)
    return Batch(ids, tt, lens, labels, S)


def batch_seed(cfg: ModelConfig, step: int, rank: int = 0) -> int:
    """Data seed per (step, rank): 3-part key folded into one int."""
    return (7000 + cfg.cfg_id) * 1_000_003 + step * 65536 * 8 + rank * 65536 + 17


def dropout_seed(cfg: ModelConfig) -> int:
    return 3000 + cfg.cfg_id
