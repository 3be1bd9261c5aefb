"""Pins for the parts of the memory oracle the round-1 review found unpinned
(VERDICT r1 "What's weak" 1):

* the persistent bytes C (oracle/memsim.persistent_bytes) -- written here as
  the DESIGN.md §3 "C (persistent)" formula, with the parameter count itself
  pinned to an independent library (HF transformers' model classes, built on
  the meta device: no weights, no network);
* the GPT-2 pre-LN event model -- closed forms for P(empty), LB, peak({L}),
  peak(first k) and the LM-head backward event, written from the DESIGN.md §3
  event order, for every BASELINE config (post-LN and pre-LN alike);
* Algorithm 1 (oracle/planner.plan) against a brute force that evaluates every
  drop set with the EVENT SIMULATOR (SURVEY c-G), not the planner's formula;
* the exact planner (reading A29) against the same simulator brute force over
  sub-layer units.
"""
import random

import numpy as np
import pytest

from oracle import estimator as oe
from oracle import memsim as om
from oracle import planner as op
from paper_conf_ipps_liaolysshfyctzlq23_b200 import workload as wl

CFGS = ["toy", "bert-base", "bert-large", "roberta-large", "gpt2-medium"]


def a16(n):
    return (n + 15) // 16 * 16


# --------------------------------------------------------------------------
# parameter counts: an independent library defines the models
# --------------------------------------------------------------------------

def _hf_count(name):
    torch = pytest.importorskip("torch")
    tr = pytest.importorskip("transformers")
    with torch.device("meta"):
        if name == "bert-base":          # BertModel + MC classifier (H -> 1)
            m, extra = tr.BertModel(tr.BertConfig()), 768 + 1
        elif name == "bert-large":       # BertForQuestionAnswering: no pooler, qa_outputs H -> 2
            c = tr.BertConfig(hidden_size=1024, num_hidden_layers=24, num_attention_heads=16,
                              intermediate_size=4096)
            m, extra = tr.BertModel(c, add_pooling_layer=False), 2 * 1024 + 2
        elif name == "roberta-large":    # RobertaModel (pooler kept for MC) + classifier H -> 1
            c = tr.RobertaConfig(vocab_size=50265, hidden_size=1024, num_hidden_layers=24,
                                 num_attention_heads=16, intermediate_size=4096,
                                 max_position_embeddings=514, type_vocab_size=1)
            m, extra = tr.RobertaModel(c), 1024 + 1
        else:                            # GPT2Model (LM head tied to wte)
            m, extra = tr.GPT2Model(tr.GPT2Config(n_embd=1024, n_layer=24, n_head=16)), 0
        return sum(p.numel() for p in m.parameters()) + extra


@pytest.mark.parametrize("name", ["bert-base", "bert-large", "roberta-large", "gpt2-medium"])
def test_param_count_equals_hf_model(name):
    assert wl.n_params(wl.CONFIGS[name]) == _hf_count(name)


@pytest.mark.parametrize("name", CFGS)
def test_persistent_bytes_formula(name):
    """DESIGN.md §3 "C (persistent)": the parameter image padded to 64 elements
    per tensor, held as weights (e), fp32 grads, fp32 master (bf16 only), AdamW
    m and v; ids and token types (4 maxT each), lengths (4 max_seqs), labels
    (8 max_seqs); 256 B of scalars; the split-K workspace 4 H^2 fp32; the
    reduction partials 296 x 2 x max(3H, F) fp32.  Each item 16-B aligned."""
    cfg = wl.CONFIGS[name]
    e = 4 if cfg.dtype == "fp32" else 2
    npad = sum(-(-int(np.prod(s)) // 64) * 64 for _, s in wl.param_spec(cfg))
    n = wl.n_params(cfg)
    assert 0 <= npad - n < 64 * len(wl.param_spec(cfg))
    copies = [e, 4, 4, 4] + ([] if cfg.dtype == "fp32" else [4])
    maxT = cfg.n_seqs * cfg.max_seq
    H, F = cfg.hidden, cfg.ffn
    C = (sum(a16(npad * c) for c in copies) + 2 * a16(4 * maxT) + a16(4 * cfg.n_seqs)
         + a16(8 * cfg.n_seqs) + 256 + a16(16 * H * H) + a16(296 * 2 * max(3 * H, F) * 4))
    assert om.persistent_bytes(cfg, cfg.n_seqs, cfg.max_seq) == C
    # 18 B/param in bf16 mode (16 in fp32) dominates C
    per_param = sum(copies)
    assert per_param == (16 if cfg.dtype == "fp32" else 18)
    assert C - per_param * n < 2 ** 27


# --------------------------------------------------------------------------
# event-model closed forms, both layer types (DESIGN.md §3 event order)
# --------------------------------------------------------------------------

def layer_bytes_per_token(cfg):
    """DESIGN.md §3 per-layer internals + output, per token (S-proportional
    parts only): post-LN QKV, O, z1(f32), h1, u, g, z2(f32), y; pre-LN a, QKV,
    O, r1(f32), m, u, g, y(f32); both = (6H + 2F) e + 8H, plus 16 B of LN
    statistics and 4h of LSE."""
    e = 4 if cfg.dtype == "fp32" else 2
    H, F, h = cfg.hidden, cfg.ffn, cfg.heads
    return (6 * H + 2 * F) * e + 8 * H + 4 * h + 16


def events(sz, dropped, L):
    """Every live-byte event value of one step for plan `dropped`, written from
    the event list of DESIGN.md §3 (not from memsim's code): forward of layer l,
    head forward (+ LM logits chunk), head backward (dy + head scratch), layer
    backward l (its internals + layer scratch), embedding backward."""
    base = sz.C + sz.e
    s = [sz.y if l in dropped else sz.a for l in range(L)]
    ev = {}
    for l in range(L):
        ev[("fwd", l)] = base + sum(s[:l]) + sz.a
        ev[("bwd", l)] = base + sum(s[:l]) + sz.i + sz.dy + sz.layer_scratch
    ev["head_fwd"] = base + sum(s) + sz.hd + sz.head_fwd_scratch
    ev["head_bwd"] = base + sum(s) + sz.hd + sz.dy + sz.head_scratch
    ev["emb_bwd"] = base + sz.dy + sz.emb_scratch
    return ev


@pytest.mark.parametrize("name", CFGS)
def test_event_closed_forms_every_config(name):
    cfg = wl.CONFIGS[name]
    L = cfg.n_layers
    for S in sorted({cfg.seq_lo, wl.roundup((cfg.seq_lo + cfg.seq_hi) // 2, cfg.pad), cfg.max_seq}):
        sz = om.sizes(cfg, cfg.n_seqs, S)
        T = cfg.n_seqs * S
        assert sz.a == T * layer_bytes_per_token(cfg)
        # P(empty), LB, peak({L}) and peak(first k) as maxima of the listed events
        P0 = max(events(sz, set(), L).values())
        assert om.no_ckpt_peak(sz) == P0
        LB = max(events(sz, set(range(L)), L).values())
        assert om.lower_bound(sz) == LB
        assert om.peak(sz, [L - 1]) == max(events(sz, {L - 1}, L).values())
        for k in range(L):
            assert om.peak(sz, range(k)) == max(events(sz, set(range(k)), L).values())
        # the collector (every layer dropped in its backward) peaks at LB
        assert om.collect_samples(sz)["peak"] == max(LB, max(events(sz, set(), L)[("fwd", l)]
                                                             - l * sz.i for l in range(L)))


def test_gpt2_lm_head_backward_event_dominates():
    """GPT-2 medium: the LM head's backward holds the fp32 logits chunk and its
    bf16 gradient (2048 tokens x padded vocab) on top of every
    saved layer, so its event sets P(empty); dropping the last layer (saving
    i bytes at that event) is then NOT a no-op, unlike Fig. 9's encoder case
    (reading A12's last resort)."""
    cfg = wl.CONFIGS["gpt2-medium"]
    L = cfg.n_layers
    VP = (cfg.vocab + 7) // 8 * 8
    for S in (256, 512, 1024):
        sz = om.sizes(cfg, cfg.n_seqs, S)
        T = cfg.n_seqs * S
        assert sz.head_scratch == a16(2048 * VP * 4) + a16(2048 * VP * 2)
        assert sz.head_fwd_scratch == a16(2048 * VP * 4)
        assert sz.hd == a16(T * 1024 * 2) + 2 * a16(8 * T)           # hf, stf, (lse, nll)
        ev = events(sz, set(), L)
        assert max(ev, key=ev.get) == "head_bwd"
        P0 = sz.C + sz.e + L * sz.a + sz.hd + sz.dy + sz.head_scratch
        assert om.no_ckpt_peak(sz) == P0
        assert om.peak(sz, [L - 1]) == P0 - sz.i
        for k in range(1, L):
            assert om.peak(sz, range(k)) == P0 - k * sz.i


@pytest.mark.parametrize("name", ["toy", "bert-base", "bert-large", "roberta-large"])
def test_post_ln_last_layer_saves_nothing(name):
    """Fig. 9 / P:177 for the encoders: the layer-backward event of the last
    layer dominates, so dropping the last layer leaves the peak unchanged."""
    cfg = wl.CONFIGS[name]
    sz = om.sizes(cfg, cfg.n_seqs, cfg.max_seq)
    ev = events(sz, set(), cfg.n_layers)
    assert max(ev, key=ev.get) == ("bwd", cfg.n_layers - 1)
    assert om.peak(sz, [cfg.n_layers - 1]) == om.no_ckpt_peak(sz)


# --------------------------------------------------------------------------
# planners vs brute force over the EVENT SIMULATOR (SURVEY c-G)
# --------------------------------------------------------------------------

def small_stacks():
    yield wl.CONFIGS["toy"]
    yield wl.small_config("bert-base", n_layers=10, n_seqs=8)
    yield wl.small_config("bert-large", n_layers=8, n_seqs=2)
    yield wl.small_config("gpt2-medium", n_layers=10, n_seqs=1, vocab=5000)
    yield wl.small_config("gpt2-medium", n_layers=6, n_seqs=2)


def trained_estimator(cfg, units=False):
    coll = om.collect_samples_units if units else om.collect_samples
    samples = []
    for S in sorted({cfg.seq_lo, wl.roundup((cfg.seq_lo + cfg.seq_hi) // 2, cfg.pad), cfg.max_seq}):
        c = coll(om.sizes(cfg, cfg.n_seqs, wl.roundup(S, cfg.pad)))
        c["x"] = cfg.n_seqs * wl.roundup(S, cfg.pad)
        samples.append(c)
    return oe.Estimator(samples)


@pytest.mark.parametrize("k", range(5))
def test_greedy_equals_simulator_brute_force(k):
    """Homogeneous stacks (every BASELINE config): Algorithm 1 on the
    estimator's predictions == the cheapest feasible drop set found by
    simulating all 2^L sets, then the lowest peak, then lexicographic."""
    cfg = list(small_stacks())[k]
    L = cfg.n_layers
    est = trained_estimator(cfg)
    rng = random.Random(31 + k)
    n_ok = 0
    for S in sorted({cfg.seq_lo, cfg.max_seq, wl.roundup(rng.randint(cfg.seq_lo, cfg.seq_hi), cfg.pad)}):
        S = wl.roundup(S, cfg.pad)
        sz = om.sizes(cfg, cfg.n_seqs, S)
        lo, hi = om.lower_bound(sz), om.no_ckpt_peak(sz)
        memo = {}

        def peak_of(D):
            if D not in memo:
                memo[D] = om.peak(sz, D)
            return memo[D]

        for M in [lo - 1, lo, hi, hi - 1] + [rng.randint(lo, hi) for _ in range(4)]:
            g = op.plan(est.predict(cfg.n_seqs * S), M)
            b = op.brute_force_sim(peak_of, L, M, [1.0] * L)
            assert g[0] == b[0], (S, M)
            if g[0] == op.OK:
                assert (g[1], g[2]) == (b[1], b[2]), (S, M)
                assert om.peak(sz, g[1]) <= M
                n_ok += 1
    assert n_ok >= 6


@pytest.mark.parametrize("k", [0, 2, 4])
def test_unit_planners_vs_simulator_brute_force(k):
    """Sub-layer units (reading A30; heterogeneous series): the exact planner
    (A29) == simulator brute force; Algorithm 1 is feasible whenever a
    feasible unit set exists (optimality there is "parity unpinned")."""
    cfg = list(small_stacks())[k]
    n = 2 * cfg.n_layers
    if n > 12:
        cfg = wl.small_config(cfg.name, **{**cfg.__dict__, "n_layers": 6})
        n = 12
    est = trained_estimator(cfg, units=True)
    rng = random.Random(41 + k)
    S = cfg.max_seq
    sz = om.sizes(cfg, cfg.n_seqs, S)
    memo = {}

    def pk(D):
        key = tuple(sorted(D))
        if key not in memo:
            memo[key] = om.simulate_step_units(sz, key).peak
        return memo[key]

    lo, hi = pk(range(n)), pk([])
    for M in [lo - 1, lo, hi] + [rng.randint(lo, hi) for _ in range(5)]:
        pred = est.predict(cfg.n_seqs * S)
        b = op.brute_force_sim(pk, n, M, [1.0] * n)
        e = op.plan_exact(pred, M)
        assert e[0] == b[0]
        if b[0] == op.OK:
            assert (e[1], e[2]) == (b[1], b[2])
        g = op.plan(pred, M)
        assert g[0] == b[0]
        if g[0] == op.OK:
            assert pk(g[1]) <= M
