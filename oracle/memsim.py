"""ORACLE (test infrastructure only): the arena event model = definition of
"peak live bytes" for a (input size, plan) pair.

Paper basis:
  * P:75 (§III-A): the footprint is parameters + gradients + optimizer states
    (constant in the input size) + activations (vary with the input size).
  * P:140 (§IV-B): a dropped block keeps only its output / input between blocks;
    the shuttling collector's footprint equals Sublinear's.
  * P:177 (§IV-D, Fig. 9): checkpointing the LAST encoder gives a peak close to
    no checkpointing, because its activations are restored at once in backward
    while the others are still alive.
  * P:51 (§II-A): activations are released as soon as their gradients are
    derived.

The tensor list and event order are DESIGN.md "Memory model" (reading R-D);
every size is align16(bytes).  This module is written from that spec alone;
the GPU arena is an independent implementation of the same spec and must
report the same integers.

Pinned by: closed forms P(empty)=C+E+(L-1)a+i+Tb, LB, peak({L})=peak(empty),
peak(first k)=P(empty)-k*i, monotonicity in x (tests/test_oracle_planning.py);
the event-list closed forms of both layer types incl. GPT-2's LM-head event,
and C written from DESIGN.md §3 with the parameter count pinned to HF
transformers' own model classes (tests/test_oracle_pins.py).

Allocation-spec constants.  The byte sizes below name allocation choices of
the DESIGN.md §3 spec that the product's arena also follows: NPART reduction
partials, the 4H^2 fp32 split-K workspace, the radix-sort digit histograms
(256 x int32 per 1024-token tile) and LM_CHUNK tokens per LM-head chunk.
They define WHICH buffers a step allocates, not any arithmetic; a change to
one of them is a change of DESIGN.md §3 and its commit cites that passage.
"""
from __future__ import annotations

import dataclasses
from typing import Dict, List, Optional, Sequence

from paper_conf_ipps_liaolysshfyctzlq23_b200.workload import (
    ARCH_ENCDEC, ARCH_PRE_LN, HEAD_LM, HEAD_QA, ModelConfig, param_spec)

LM_CHUNK = 2048     # tokens per LM-head chunk (logits never exceed LM_CHUNK x Vpad)


def vpad(v: int) -> int:
    return (v + 7) // 8 * 8


def a16(n: int) -> int:
    return (int(n) + 15) // 16 * 16


def ebytes(cfg: ModelConfig) -> int:
    return 4 if cfg.dtype == "fp32" else 2


NPART = 296   # fixed count of deterministic reduction partials (DESIGN "Memory model")


def buckets(cfg: ModelConfig) -> List[List[int]]:
    """Gradient buckets as lists of parameter indices, in layout order: the
    embedding tensors, one bucket per encoder layer (12 tensors), the head
    (all-reduced / reduce-scattered as soon as each is final).
    Encoder-decoder: embedding, encoder layers, [encoder final LN + decoder
    layer 0], decoder layers (20 tensors), decoder final LN."""
    n = len(param_spec(cfg))
    if cfg.arch == ARCH_ENCDEC:
        out = [[0, 1]]
        i = 2
        for _ in range(cfg.n_layers):
            out.append(list(range(i, i + 12)))
            i += 12
        out.append(list(range(i, i + 2 + 20)))          # enc.lnf with decoder layer 0
        i += 22
        for _ in range(1, cfg.n_dec_layers):
            out.append(list(range(i, i + 20)))
            i += 20
        out.append(list(range(i, n)))
        return out
    n_emb = 2 if cfg.arch == ARCH_PRE_LN else 5
    out = [list(range(n_emb))]
    for l in range(cfg.n_layers):
        out.append(list(range(n_emb + 12 * l, n_emb + 12 * (l + 1))))
    out.append(list(range(n_emb + 12 * cfg.n_layers, n)))
    return out


def padded_numel(cfg: ModelConfig, world: int = 1, zero1: bool = False) -> int:
    """Elements of the padded flat parameter image: every tensor rounded up to
    64 elements; with ZeRO-1 every bucket rounded up to 64 x world elements so it
    splits into world equal shards."""
    spec = param_spec(cfg)
    unit = 64 * world if zero1 else 64
    tot = 0
    for b in buckets(cfg):
        nb = sum((int(_prod(spec[i][1])) + 63) // 64 * 64 for i in b)
        tot += (nb + unit - 1) // unit * unit
    return tot


def persistent_bytes(cfg: ModelConfig, max_seqs: int, max_seq_len: int, world: int = 1,
                     zero1: bool = False) -> int:
    """C: weights (e), fp32 grads, fp32 master (bf16 only), AdamW m and v (with
    ZeRO-1 master, m and v hold this rank's 1/world shard only), batch
    metadata buffers, misc, and the fixed backward workspaces."""
    e = ebytes(cfg)
    H, F = cfg.hidden, cfg.ffn
    npad = padded_numel(cfg, world, zero1)
    nsh = npad // world if zero1 else npad
    c = a16(npad * e) + a16(npad * 4) + a16(nsh * 4) + a16(nsh * 4)     # w, grad, m, v
    if cfg.dtype != "fp32":
        c += a16(nsh * 4)                                                # master
    maxT = max_seqs * max_seq_len
    c += a16(maxT * 4) * 2 + a16(max_seqs * 4) + a16(2 * max_seqs * 4)  # ids, tt, lens, labels
    c += a16(256)                                                        # misc scalars
    c += a16(4 * H * H * 4)                                              # wgrad split-K workspace
    c += a16(NPART * 2 * max(3 * H, F) * 4)                              # LN / bias partials
    return c


def _prod(s):
    n = 1
    for v in s:
        n *= v
    return n


@dataclasses.dataclass(frozen=True)
class Sizes:
    """Byte sizes of every arena object for one input shape (B, S)."""
    C: int
    E: List[int]          # embedding-forward objects (z0, st0, x1)
    internals: List[int]  # one layer's saved internals
    y: int                # layer output
    head: List[int]       # head-forward objects
    dy: int               # backward gradient buffer
    head_scratch: int
    layer_scratch: int
    emb_scratch: int
    n_layers: int
    head_fwd_scratch: int = 0   # transient during the head forward (LM logits chunk)
    per_layer: Optional[List[List[int]]] = None   # heterogeneous stages: internals of each layer

    def ints(self, l: int) -> List[int]:
        """Internals of layer l (they differ by stage only in the FFN tensors u, g)."""
        return self.per_layer[l] if self.per_layer is not None else self.internals

    @property
    def i(self) -> int:
        return sum(self.internals)

    @property
    def a(self) -> int:
        return self.i + self.y

    @property
    def e(self) -> int:
        return sum(self.E)

    @property
    def hd(self) -> int:
        return sum(self.head)


def sizes(cfg: ModelConfig, B: int, S: int, max_seqs: Optional[int] = None,
          max_seq_len: Optional[int] = None, world: int = 1, zero1: bool = False) -> Sizes:
    e = ebytes(cfg)
    H, F, h = cfg.hidden, cfg.ffn, cfg.heads
    T = B * S
    ms = cfg.n_seqs if max_seqs is None else max_seqs
    mx = cfg.max_seq if max_seq_len is None else max_seq_len
    # pre-LN sums z0, z1, z2 are fp32 in every mode (reading R-P: bf16 z loses
    # the row mean/spread balance that LayerNorm's backward needs)
    pre = cfg.arch == ARCH_PRE_LN
    def layer_ints(Fl: int) -> List[int]:
        if pre:
            # GPT-2: the residual stream (x1, r1, y) is fp32; LN outputs a, m are the GEMM operands
            return [a16(T * H * e), a16(T * 8), a16(T * 3 * H * e),          # a, st1, QKV
                    a16(T * H * e), a16(B * h * S * 4),                       # O, LSE
                    a16(T * H * 4), a16(T * 8), a16(T * H * e),               # r1, st2, m
                    a16(T * Fl * e), a16(T * Fl * e)]                         # u, g
        return [a16(T * 3 * H * e), a16(T * H * e), a16(B * h * S * 4),     # QKV, O, LSE
                a16(T * H * 4), a16(T * 8), a16(T * H * e),                   # z1, st1, h1
                a16(T * Fl * e), a16(T * Fl * e),                             # u, g
                a16(T * H * 4), a16(T * 8)]                                   # z2, st2
    # (heterogeneous stages: layer l's u, g use its own FFN width;
    #  the backward layer scratch below is sized for the widest, F = cfg.ffn)
    if pre:
        E = [a16(T * H * 4)]                                                   # x1
        y = a16(T * H * 4)
    else:
        # pre-LN sums z0, z1, z2 are fp32 in every mode (reading R-P: bf16 z loses
        # the row mean/spread balance that LayerNorm's backward needs)
        E = [a16(T * H * 4), a16(T * 8), a16(T * H * e)]                       # z0, st0, x1
        y = a16(T * H * e)
    internals = layer_ints(cfg.ffn_of(0))
    per_layer = [layer_ints(cfg.ffn_of(l)) for l in range(cfg.n_layers)] if cfg.ffn_layers else None
    head_fwd = 0
    if cfg.head == HEAD_LM:
        VP = vpad(cfg.vocab)
        head = [a16(T * H * e), a16(T * 8), a16(T * 8)]                       # hf, stf, (lse, nll)
        head_fwd = a16(LM_CHUNK * VP * 4)                                      # fp32 logits chunk
        head_scr = a16(LM_CHUNK * VP * 4) + a16(LM_CHUNK * VP * e)             # logits, dlogits
    elif cfg.head == HEAD_QA:
        head = [a16(T * 2 * 4)]
        head_scr = a16(T * 2 * 4)
    else:
        head = [a16(B * H * e), a16(B * cfg.n_out * 4)]                       # pooled, logits
        head_scr = a16(B * cfg.n_out * 4) + a16(B * H * 4) * 2
    dy = a16(T * H * 4)
    layer_scr = a16(T * H * 4) + a16(T * F * e) + a16(T * 3 * H * e) + a16(B * h * S * 4)
    ntiles = (ms * mx + 1023) // 1024
    emb_scr = a16(T * H * 4) + a16(16 * T) + a16(4 * 256 * ntiles)   # dz0, 4 int32[T] sort arrays, digit histograms
    return Sizes(persistent_bytes(cfg, ms, mx, world, zero1), E, internals, y, head, dy, head_scr,
                 layer_scr, emb_scr, cfg.n_layers, head_fwd, per_layer)


# --------------------------------------------------------------------------
# event-level simulator
# --------------------------------------------------------------------------

class Arena:
    """Two-ended accounting: a LIFO stack (activations) and a LIFO top region
    (transients).  live = C + stack + top.  Frees must be LIFO per region."""

    def __init__(self, C: int):
        self.C = C
        self.stack: List[int] = []
        self.top: List[int] = []
        self.peak = C
        self.timeline: List[int] = [C]
        self.top_peak_phase = 0

    @property
    def live(self) -> int:
        return self.C + sum(self.stack) + sum(self.top)

    def _tick(self):
        v = self.live
        self.timeline.append(v)
        self.peak = max(self.peak, v)
        self.top_peak_phase = max(self.top_peak_phase, sum(self.top))

    def push(self, n):
        self.stack.append(n)
        self._tick()

    def pop(self, n):
        assert self.stack and self.stack[-1] == n, "stack free out of LIFO order"
        self.stack.pop()
        self.timeline.append(self.live)

    def talloc(self, n):
        self.top.append(n)
        self._tick()

    def tfree(self, n):
        assert self.top and self.top[-1] == n, "top free out of LIFO order"
        self.top.pop()
        self.timeline.append(self.live)


def simulate_step(sz: Sizes, dropped: Sequence[int]) -> Arena:
    """One training step (forward, backward) under a plan of dropped layers
    (0-based).  Returns the arena with its peak and timeline."""
    L = sz.n_layers
    drop = set(dropped)
    A = Arena(sz.C)
    for t in sz.E:
        A.push(t)
    for l in range(L):                                   # forward
        if l in drop:                                    # no-save: internals transient
            for t in sz.ints(l):
                A.talloc(t)
            A.push(sz.y)
            for t in reversed(sz.ints(l)):
                A.tfree(t)
        else:
            for t in sz.ints(l):
                A.push(t)
            A.push(sz.y)
    for t in sz.head:
        A.push(t)
    if sz.head_fwd_scratch:                              # LM logits chunk (head forward)
        A.talloc(sz.head_fwd_scratch)
        A.tfree(sz.head_fwd_scratch)
    A.talloc(sz.dy)                                      # backward
    A.talloc(sz.head_scratch)
    A.tfree(sz.head_scratch)
    for t in reversed(sz.head):
        A.pop(t)
    A.pop(sz.y)                                          # y_L
    for l in reversed(range(L)):
        if l in drop:                                    # recompute before gradients
            for t in sz.ints(l):
                A.push(t)
        A.talloc(sz.layer_scratch)
        A.tfree(sz.layer_scratch)
        for t in reversed(sz.ints(l)):
            A.pop(t)
        if l > 0:
            A.pop(sz.y)                                  # y_{l-1}: input of layer l
    A.talloc(sz.emb_scratch)
    A.tfree(sz.emb_scratch)
    for t in reversed(sz.E):
        A.pop(t)
    A.tfree(sz.dy)
    assert A.live == sz.C
    return A


def peak(sz: Sizes, dropped: Sequence[int]) -> int:
    return simulate_step(sz, dropped).peak


def no_ckpt_peak(sz: Sizes) -> int:
    return peak(sz, [])


def lower_bound(sz: Sizes) -> int:
    """LB: every layer dropped.  For post-LN stacks this equals dropping all but
    the last (the last saves nothing at the layer-backward peak); when the
    head-backward event dominates (GPT-2's LM head) dropping the last layer too
    lowers it (reading A12's last resort)."""
    return peak(sz, range(sz.n_layers))


# --------------------------------------------------------------------------
# shuttling collector (Fig. 7): what a sheltered iteration measures
# --------------------------------------------------------------------------

def collect_samples(sz: Sizes) -> Dict[str, object]:
    """Per-layer deltas of the two forward passes (pass 1 save-mode -> a_l,
    pass 2 no-save -> y_l), embedding / head deltas, and the backward
    transient maxima per phase, all in arena bytes; plus the collector's own
    peak (the sheltered iteration drops every layer)."""
    L = sz.n_layers
    A = Arena(sz.C)
    base = A.live
    for t in sz.E:
        A.push(t)
    E = A.live - base
    a, y = [], []
    for l in range(L):
        b0 = A.live
        for t in sz.ints(l):                             # pass 1: normal forward
            A.push(t)
        A.push(sz.y)
        a.append(A.live - b0)
        A.pop(sz.y)
        for t in reversed(sz.ints(l)):                   # discard output + activations
            A.pop(t)
        for t in sz.ints(l):                             # pass 2: keep only the output
            A.talloc(t)
        A.push(sz.y)
        for t in reversed(sz.ints(l)):
            A.tfree(t)
        y.append(A.live - b0)
    b0 = A.live
    for t in sz.head:
        A.push(t)
    hd = A.live - b0
    if sz.head_fwd_scratch:
        A.talloc(sz.head_fwd_scratch)
        A.tfree(sz.head_fwd_scratch)
    # backward with every layer recomputed; per-phase max of the top region
    A.talloc(sz.dy)
    A.top_peak_phase = sum(A.top)
    A.talloc(sz.head_scratch)
    A.tfree(sz.head_scratch)
    th = A.top_peak_phase
    for t in reversed(sz.head):
        A.pop(t)
    A.pop(sz.y)
    A.top_peak_phase = sum(A.top)
    for l in reversed(range(L)):
        for t in sz.ints(l):
            A.push(t)
        A.talloc(sz.layer_scratch)
        A.tfree(sz.layer_scratch)
        for t in reversed(sz.ints(l)):
            A.pop(t)
        if l > 0:
            A.pop(sz.y)
    tb = A.top_peak_phase
    A.top_peak_phase = sum(A.top)
    A.talloc(sz.emb_scratch)
    A.tfree(sz.emb_scratch)
    te = A.top_peak_phase
    for t in reversed(sz.E):
        A.pop(t)
    A.tfree(sz.dy)
    return dict(C=sz.C, E=E, a=a, y=y, Hd=hd, Th=th, Tb=tb, Te=te, peak=A.peak)


# --------------------------------------------------------------------------
# sub-layer checkpoint units (DESIGN reading A30)
# --------------------------------------------------------------------------
# P:125 and P:140 name the "attention block" as a unit Mimose can checkpoint
# ("the output ... of the attention block"), P:170 lets a stage be any
# user-code structure.  With granularity 1 each layer l is two units:
#   unit 2l   attention block  post-LN: QKV, O, LSE, z1, st1 -> h1; pre-LN: a, st1, QKV, O, LSE -> r1
#   unit 2l+1 FFN block        post-LN: u, g, z2, st2 -> y;     pre-LN: st2, m, u, g -> y
# Forward: a kept unit pushes its internals then its output; a dropped unit
# places its internals in the top region, pushes its output, frees them.
# Backward of layer l (after y_l is gone):
#   FFN dropped -> push its internals (recompute from h1 / r1)
#   talloc layer scratch; FFN-block gradients; pop FFN internals; pop h1 / r1
#   attention dropped -> push its internals (recompute from y_{l-1})
#   attention-block gradients; tfree scratch; pop attention internals; pop y_{l-1}
# With nothing dropped the event sequence reaches the same peak as the layer
# model (same push order), and the planner's position-aware peak applies
# unchanged to the 2L-unit series.

def unit_list(sz: Sizes) -> List[tuple]:
    """[(internals, output)] for the 2L units of a stack (both layer types keep
    10 internals whose 6th is the block boundary h1 / r1)."""
    assert len(sz.internals) == 10
    out = []
    for l in range(sz.n_layers):
        ints = sz.ints(l)
        out += [(ints[:5], ints[5]), (ints[6:], sz.y)]
    return out


def _unit_forward(A: Arena, units, drop) -> None:
    for u, (ints, o) in enumerate(units):
        if u in drop:
            for t in ints:
                A.talloc(t)
            A.push(o)
            for t in reversed(ints):
                A.tfree(t)
        else:
            for t in ints:
                A.push(t)
            A.push(o)


def _unit_backward_layers(A: Arena, sz: Sizes, units, drop) -> None:
    L = sz.n_layers
    for l in reversed(range(L)):
        (att, h1), (ffn, _) = units[2 * l], units[2 * l + 1]
        if 2 * l + 1 in drop:                        # recompute the FFN block from h1
            for t in ffn:
                A.push(t)
        A.talloc(sz.layer_scratch)
        for t in reversed(ffn):                      # FFN-block gradients done
            A.pop(t)
        A.pop(h1)
        if 2 * l in drop:                            # recompute the attention block from y_{l-1}
            for t in att:
                A.push(t)
        A.tfree(sz.layer_scratch)                    # attention-block gradients done
        for t in reversed(att):
            A.pop(t)
        if l > 0:
            A.pop(sz.y)


def simulate_step_units(sz: Sizes, dropped: Sequence[int]) -> Arena:
    """One training step under a plan over the 2L sub-layer units (0-based)."""
    units = unit_list(sz)
    drop = set(dropped)
    A = Arena(sz.C)
    for t in sz.E:
        A.push(t)
    _unit_forward(A, units, drop)
    for t in sz.head:
        A.push(t)
    if sz.head_fwd_scratch:
        A.talloc(sz.head_fwd_scratch)
        A.tfree(sz.head_fwd_scratch)
    A.talloc(sz.dy)
    A.talloc(sz.head_scratch)
    A.tfree(sz.head_scratch)
    for t in reversed(sz.head):
        A.pop(t)
    A.pop(sz.y)
    _unit_backward_layers(A, sz, units, drop)
    A.talloc(sz.emb_scratch)
    A.tfree(sz.emb_scratch)
    for t in reversed(sz.E):
        A.pop(t)
    A.tfree(sz.dy)
    assert A.live == sz.C
    return A


def collect_samples_units(sz: Sizes) -> Dict[str, object]:
    """The shuttling collector over units: per unit, pass 1 (save mode) -> a_u,
    pass 2 (no-save) -> y_u; the sheltered backward recomputes every unit."""
    units = unit_list(sz)
    A = Arena(sz.C)
    base = A.live
    for t in sz.E:
        A.push(t)
    E = A.live - base
    a, y = [], []
    for ints, o in units:
        b0 = A.live
        for t in ints:
            A.push(t)
        A.push(o)
        a.append(A.live - b0)
        A.pop(o)
        for t in reversed(ints):
            A.pop(t)
        for t in ints:
            A.talloc(t)
        A.push(o)
        for t in reversed(ints):
            A.tfree(t)
        y.append(A.live - b0)
    b0 = A.live
    for t in sz.head:
        A.push(t)
    hd = A.live - b0
    if sz.head_fwd_scratch:
        A.talloc(sz.head_fwd_scratch)
        A.tfree(sz.head_fwd_scratch)
    A.talloc(sz.dy)
    A.top_peak_phase = sum(A.top)
    A.talloc(sz.head_scratch)
    A.tfree(sz.head_scratch)
    th = A.top_peak_phase
    for t in reversed(sz.head):
        A.pop(t)
    A.pop(sz.y)
    A.top_peak_phase = sum(A.top)
    _unit_backward_layers(A, sz, units, set(range(len(units))))
    tb = A.top_peak_phase
    A.top_peak_phase = sum(A.top)
    A.talloc(sz.emb_scratch)
    A.tfree(sz.emb_scratch)
    te = A.top_peak_phase
    for t in reversed(sz.E):
        A.pop(t)
    A.tfree(sz.dy)
    return dict(C=sz.C, E=E, a=a, y=y, Hd=hd, Th=th, Tb=tb, Te=te, peak=A.peak)


# --------------------------------------------------------------------------
# encoder-decoder (reading A32): DESIGN.md §3 "Encoder-decoder"
# --------------------------------------------------------------------------

@dataclasses.dataclass(frozen=True)
class EncDecSizes:
    C: int
    E: List[int]          # x1_s
    enc_ints: List[int]
    enc_y: int
    bundle: List[int]     # output of the last encoder unit: x_L, enc_out, enc_st, x1_t
    dec_ints: List[int]
    dec_y: int
    head: List[int]
    head_fwd_scratch: int
    head_scratch: int
    dy: int
    denc: int
    layer_scratch: int    # uniform over both stacks: decoder + cross + encoder parts
    emb_scratch: int      # uniform over both embeddings
    n_enc: int
    n_dec: int

    def ints(self, u):
        return self.enc_ints if u < self.n_enc else self.dec_ints

    def outs(self, u):
        if u < self.n_enc - 1:
            return [self.enc_y]
        if u == self.n_enc - 1:
            return self.bundle
        return [self.dec_y]


def sizes_encdec(cfg: ModelConfig, B: int, Ss: int, St: int, max_seqs: Optional[int] = None,
                 max_seq_len: Optional[int] = None, world: int = 1, zero1: bool = False) -> EncDecSizes:
    e = ebytes(cfg)
    H, F, h = cfg.hidden, cfg.ffn, cfg.heads
    Ts, Tt = B * Ss, B * St
    ms = cfg.n_seqs if max_seqs is None else max_seqs
    mx = cfg.max_seq if max_seq_len is None else max_seq_len

    def pre_ints(T, S):     # a, st1, QKV, O, LSE, r1, st2, m, u, g (GPT-2 layer order)
        return [a16(T * H * e), a16(T * 8), a16(T * 3 * H * e), a16(T * H * e), a16(B * h * S * 4),
                a16(T * H * 4), a16(T * 8), a16(T * H * e), a16(T * F * e), a16(T * F * e)]

    dec = [a16(Tt * H * e), a16(Tt * 8), a16(Tt * 3 * H * e), a16(Tt * H * e), a16(B * h * St * 4),  # a st1 QKV O LSE
           a16(Tt * H * 4), a16(Tt * 8), a16(Tt * H * e), a16(Tt * H * e), a16(Ts * 2 * H * e),    # r1 st2 c Qc KVc
           a16(Tt * H * e), a16(B * h * St * 4), a16(Tt * H * 4), a16(Tt * 8), a16(Tt * H * e),    # Oc LSEc r2 st3 m
           a16(Tt * F * e), a16(Tt * F * e)]                                                         # u g

    def lscr(T, S):
        return a16(T * H * 4) + a16(T * F * e) + a16(T * 3 * H * e) + a16(B * h * S * 4)

    ntiles = (ms * mx + 1023) // 1024

    def escr(T):
        return a16(T * H * 4) + a16(16 * T) + a16(4 * 256 * ntiles)

    VP = vpad(cfg.vocab)
    return EncDecSizes(
        persistent_bytes(cfg, ms, mx, world, zero1), [a16(Ts * H * 4)], pre_ints(Ts, Ss), a16(Ts * H * 4),
        [a16(Ts * H * 4), a16(Ts * H * e), a16(Ts * 8), a16(Tt * H * 4)], dec, a16(Tt * H * 4),
        [a16(Tt * H * e), a16(Tt * 8), a16(Tt * 8)], a16(LM_CHUNK * VP * 4),
        a16(LM_CHUNK * VP * 4) + a16(LM_CHUNK * VP * e), a16(Tt * H * 4), a16(Ts * H * 4),
        lscr(Tt, St) + a16(Ts * 2 * H * e) + lscr(Ts, Ss), escr(Ts) + escr(Tt),
        cfg.n_layers, cfg.n_dec_layers)


def _encdec_forward(A: Arena, sz: EncDecSizes, drop, collect=False):
    a_s, y_s = [], []
    for u in range(sz.n_enc + sz.n_dec):
        b0 = A.live
        ints, outs = sz.ints(u), sz.outs(u)
        if collect:                                           # pass 1: save mode, then discarded
            for t in ints:
                A.push(t)
            for t in outs:
                A.push(t)
            a_s.append(A.live - b0)
            for t in reversed(outs):
                A.pop(t)
            for t in reversed(ints):
                A.pop(t)
        if collect or u in drop:
            for t in ints:
                A.talloc(t)
            for t in outs:
                A.push(t)
            for t in reversed(ints):
                A.tfree(t)
        else:
            for t in ints:
                A.push(t)
            for t in outs:
                A.push(t)
        y_s.append(A.live - b0)
    return a_s, y_s


def _encdec_backward(A: Arena, sz: EncDecSizes, drop, phases=None):
    Le, Ld = sz.n_enc, sz.n_dec
    A.talloc(sz.denc)
    A.talloc(sz.dy)
    A.top_peak_phase = sum(A.top)
    A.talloc(sz.head_scratch)
    A.tfree(sz.head_scratch)
    th = A.top_peak_phase
    for t in reversed(sz.head):
        A.pop(t)
    A.pop(sz.dec_y)                                          # the last decoder unit's output
    A.top_peak_phase = sum(A.top)
    for j in reversed(range(Ld)):
        u = Le + j
        if u in drop:
            for t in sz.dec_ints:
                A.push(t)
        A.talloc(sz.layer_scratch)
        A.tfree(sz.layer_scratch)
        for t in reversed(sz.dec_ints):
            A.pop(t)
        if j > 0:
            A.pop(sz.dec_y)
    tb = A.top_peak_phase
    A.top_peak_phase = sum(A.top)
    A.talloc(sz.emb_scratch)                                 # decoder embedding backward
    A.tfree(sz.emb_scratch)
    te = A.top_peak_phase
    x_L, enc_out, enc_st, x1_t = sz.bundle
    A.pop(x1_t)
    A.pop(enc_st)                                            # encoder final LN backward (in place, no scratch)
    A.pop(enc_out)
    A.pop(x_L)
    A.top_peak_phase = sum(A.top)
    for l in reversed(range(Le)):
        if l in drop:
            for t in sz.enc_ints:
                A.push(t)
        A.talloc(sz.layer_scratch)
        A.tfree(sz.layer_scratch)
        for t in reversed(sz.enc_ints):
            A.pop(t)
        if l > 0:
            A.pop(sz.enc_y)
    tb = max(tb, A.top_peak_phase)
    A.top_peak_phase = sum(A.top)
    A.talloc(sz.emb_scratch)                                 # encoder embedding backward
    A.tfree(sz.emb_scratch)
    te = max(te, A.top_peak_phase)
    for t in reversed(sz.E):
        A.pop(t)
    A.tfree(sz.dy)
    A.tfree(sz.denc)
    if phases is not None:
        phases.update(Th=th, Tb=tb, Te=te)


def simulate_step_encdec(sz: EncDecSizes, dropped: Sequence[int]) -> Arena:
    """One encoder-decoder step under a plan over the Le + Ld units (encoder l,
    decoder Le + j)."""
    drop = set(dropped)
    A = Arena(sz.C)
    for t in sz.E:
        A.push(t)
    _encdec_forward(A, sz, drop)
    for t in sz.head:
        A.push(t)
    A.talloc(sz.head_fwd_scratch)
    A.tfree(sz.head_fwd_scratch)
    _encdec_backward(A, sz, drop)
    assert A.live == sz.C
    return A


def collect_samples_encdec(sz: EncDecSizes) -> Dict[str, object]:
    """The shuttling collector over the Le + Ld units (every unit dropped in the
    sheltered backward)."""
    A = Arena(sz.C)
    for t in sz.E:
        A.push(t)
    E = A.live - sz.C
    a, y = _encdec_forward(A, sz, set(), collect=True)
    b0 = A.live
    for t in sz.head:
        A.push(t)
    hd = A.live - b0
    A.talloc(sz.head_fwd_scratch)
    A.tfree(sz.head_fwd_scratch)
    ph = {}
    _encdec_backward(A, sz, set(range(sz.n_enc + sz.n_dec)), ph)
    return dict(C=sz.C, E=E, a=a, y=y, Hd=hd, Th=ph["Th"], Tb=ph["Tb"], Te=ph["Te"], peak=A.peak)
