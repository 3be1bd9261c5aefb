"""Pins for oracle/philox.py, memsim.py, estimator.py, planner.py (CPU)."""
import os
import random

import numpy as np
import pytest

from oracle import estimator as oe
from oracle import memsim as om
from oracle import philox as px
from oracle import planner as op
from paper_conf_ipps_liaolysshfyctzlq23_b200 import workload as wl

GOLD = os.path.join(os.path.dirname(__file__), "golden")


# ------------------------------------------------------------- Philox -----

def test_philox_known_answers():
    n = 0
    for line in open(os.path.join(GOLD, "philox_kat.txt")):
        if line.startswith("#") or not line.strip():
            continue
        w = [int(t, 16) for t in line.split()]
        out = px.philox4x32_10(*w[:4], w[4], w[5])
        assert [int(o) for o in out] == w[6:], line
        n += 1
    assert n == 3


def test_keep_rate_within_4_sigma():
    n, p = 10_000_000, 0.1
    keep = px.keep_mask(n, p, seed=3001, site=px.site_word(px.KIND_FFN_OUT, 7), step=5)
    rate = keep.mean()
    sigma = np.sqrt(p * (1 - p) / n)
    assert abs(rate - (1 - p)) < 4 * sigma
    assert px.keep_threshold(0.1) == 3865470566


def test_sites_do_not_collide():
    seen = set()
    for rank in range(3):
        for layer in list(range(24)) + [px.LAYER_NONE]:
            for kind in range(5):
                s = px.site_word(kind, layer, rank)
                assert s not in seen
                seen.add(s)


# ------------------------------------------------------------- memsim -----

CFGS = ["toy", "bert-base", "bert-large", "roberta-large", "gpt2-medium"]
POST_LN = ["toy", "bert-base", "bert-large", "roberta-large"]


def cfg_sizes(name, S):
    cfg = wl.CONFIGS[name]
    return cfg, om.sizes(cfg, cfg.n_seqs, S)


@pytest.mark.parametrize("name", POST_LN)
def test_memsim_closed_forms(name):
    cfg = wl.CONFIGS[name]
    for S in (cfg.seq_lo, (cfg.seq_lo + cfg.seq_hi) // 2 // cfg.pad * cfg.pad or cfg.pad, cfg.max_seq):
        sz = om.sizes(cfg, cfg.n_seqs, S)
        L = cfg.n_layers
        Tb = sz.dy + sz.layer_scratch
        P0 = sz.C + sz.e + (L - 1) * sz.a + sz.i + Tb
        LB = sz.C + sz.e + (L - 1) * sz.y + sz.i + Tb
        assert om.no_ckpt_peak(sz) == P0
        assert om.peak(sz, range(L)) == LB
        assert om.lower_bound(sz) == LB
        assert om.peak(sz, [L - 1]) == P0            # Fig. 9 / P:177: last layer saves nothing
        for k in range(L):
            assert om.peak(sz, range(k)) == P0 - k * sz.i
        coll = om.collect_samples(sz)
        assert coll["peak"] == LB                     # P:140 collector footprint == Sublinear's


@pytest.mark.parametrize("name", CFGS)
def test_memsim_monotone_in_x(name):
    cfg = wl.CONFIGS[name]
    rng = random.Random(1)
    for _ in range(5):
        plan = sorted(rng.sample(range(cfg.n_layers), rng.randint(0, cfg.n_layers)))
        prev = 0
        for S in range(cfg.pad, cfg.max_seq + 1, cfg.pad):
            pk = om.peak(om.sizes(cfg, cfg.n_seqs, S), plan)
            assert pk >= prev
            prev = pk


@pytest.mark.parametrize("name", CFGS)
def test_collected_series_and_predicted_peak_formula(name):
    """The planner's position-aware peak formula == the event simulator."""
    cfg = wl.CONFIGS[name]
    rng = random.Random(2)
    for S in (cfg.seq_lo, cfg.max_seq):
        sz = om.sizes(cfg, cfg.n_seqs, S)
        c = om.collect_samples(sz)
        assert c["a"] == [sz.a] * cfg.n_layers and c["y"] == [sz.y] * cfg.n_layers
        assert c["E"] == sz.e and c["Hd"] == sz.hd
        assert c["Tb"] == sz.dy + sz.layer_scratch
        assert c["Th"] == sz.dy + sz.head_scratch and c["Te"] == sz.dy + sz.emb_scratch
        for _ in range(10):
            plan = rng.sample(range(cfg.n_layers), rng.randint(0, cfg.n_layers))
            assert op.predicted_peak(c, plan) == om.peak(sz, plan)


def test_bert_base_saved_bytes_per_token():
    """SURVEY §8(a) a7 layout with the pre-LN sums z1, z2 in fp32 (reading R-P):
    (6H + 2F) e + 2*4H + 4h + 16 bytes per token per kept layer."""
    cfg = wl.CONFIGS["bert-base"]
    sz = om.sizes(cfg, 64, 128)
    T = 64 * 128
    assert sz.a == T * ((6 * 768 + 2 * 3072) * 2 + 2 * 4 * 768 + 4 * 12 + 16)


# ---------------------------------------------------------- estimator -----

@pytest.mark.parametrize("name", CFGS)
def test_estimator_exact_on_integer_quadratics(name):
    cfg = wl.CONFIGS[name]
    rng = np.random.default_rng(7)
    xs_all = [cfg.n_seqs * S for S in range(cfg.pad, cfg.max_seq + 65, cfg.pad)]
    for _ in range(50):
        c0, c1, c2 = (int(v) for v in rng.integers(0, 10**9, 3))
        c1 //= 1000
        c2 //= 10**6
        f = lambda x: c0 + c1 * x + c2 * x * x
        xs = rng.choice([x for x in xs_all if x <= cfg.n_seqs * cfg.max_seq], size=10)
        q = oe.Quadratic(xs, [f(int(x)) for x in xs])
        if len(set(xs.tolist())) >= 3:
            assert q.margin == 0
            for x in xs_all:                       # interpolation and extrapolation
                assert q.predict(x) == f(x)


def test_estimator_linear_constant_and_fallback():
    xs = [100, 200, 300, 400]
    q = oe.Quadratic(xs, [7 + 3 * x for x in xs])
    assert q.predict(1000) == 3007
    q = oe.Quadratic(xs, [42] * 4)
    assert q.predict(10) == 42
    q = oe.Quadratic([100, 100, 200], [5, 5, 9])       # 2 distinct -> degree 1
    assert q.degree == 1 and q.predict(300) == 13
    q = oe.Quadratic([100, 100], [5, 5])               # 1 distinct -> constant
    assert q.degree == 0 and q.predict(999) == 5
    q = oe.Quadratic([1, 2, 3, 4], [0, 10, 0, 10])      # noisy: margin covers residuals
    for x, y in zip([1, 2, 3, 4], [0, 10, 0, 10]):
        assert q.predict(x) >= y


@pytest.mark.parametrize("name", CFGS)
def test_estimator_on_collected_series_is_exact(name):
    cfg = wl.CONFIGS[name]
    rng = random.Random(3)
    Ss = sorted(rng.sample(range(cfg.pad, cfg.max_seq + 1, cfg.pad), 5))
    samples = []
    for S in Ss:
        c = om.collect_samples(om.sizes(cfg, cfg.n_seqs, S))
        c["x"] = cfg.n_seqs * S
        samples.append(c)
    est = oe.Estimator(samples)
    for S in range(cfg.pad, cfg.max_seq + 1, cfg.pad):
        truth = om.collect_samples(om.sizes(cfg, cfg.n_seqs, S))
        pred = est.predict(cfg.n_seqs * S)
        for k in ("E", "Hd", "Th", "Tb", "Te", "a", "y"):
            assert pred[k] == truth[k], (k, S)


# ------------------------------------------------------------ planner -----

def parse_traces():
    rows = []
    for line in open(os.path.join(GOLD, "alg1_traces.txt")):
        if line.startswith("#") or not line.strip():
            continue
        est, exc, bk, st, dr = [t.strip() for t in line.split("|")]
        rows.append(([int(v) for v in est.split(",")], int(exc),
                     [[int(v) for v in b.split(",")] for b in bk.split(";")],
                     st, [int(v) for v in dr.split(",")] if dr else []))
    return rows


@pytest.mark.parametrize("row", parse_traces())
def test_algorithm1_hand_traces(row):
    est, excess, buckets, status, dropped = row
    st, chosen, bks = op.greedy_core(est, excess)
    assert bks == buckets
    assert st == status
    assert chosen == dropped


def random_stack(rng, L, homogeneous):
    C = rng.randint(0, 1000)
    if homogeneous:
        y = rng.randint(1, 50)
        a = [y + rng.randint(1, 200)] * L
        ys = [y] * L
    else:
        ys = [rng.randint(1, 50) for _ in range(L)]
        a = [ys[l] + rng.randint(1, 200) for l in range(L)]
    return dict(C=C, E=rng.randint(1, 100), a=a, y=ys, Hd=rng.randint(0, 20),
                Th=rng.randint(1, 100), Tb=rng.randint(50, 400), Te=rng.randint(1, 300))


def test_greedy_equals_brute_force_on_homogeneous_stacks():
    rng = random.Random(11)
    n = 0
    for _ in range(600):
        L = rng.randint(1, 10)
        p = random_stack(rng, L, True)
        lo, hi = op.predicted_peak(p, range(L)), op.predicted_peak(p, [])
        M = rng.randint(lo - 5, hi + 5)
        g = op.plan(p, M)
        b = op.brute_force(p, M, [1.0] * L)
        assert g[0] == b[0]
        if g[0] == op.OK:
            assert g[1] == b[1] and g[2] == b[2] <= M
            n += 1
    assert n > 300


def test_greedy_feasible_on_heterogeneous_stacks():
    rng = random.Random(12)
    opt = tot = 0
    for _ in range(600):
        L = rng.randint(1, 10)
        p = random_stack(rng, L, False)
        lo, hi = op.predicted_peak(p, range(L)), op.predicted_peak(p, [])
        M = rng.randint(lo - 5, hi + 5)
        cost = [float(p["a"][l]) for l in range(L)]
        g = op.plan(p, M)
        b = op.brute_force(p, M, cost)
        assert g[0] == b[0]                      # never infeasible when a plan exists
        if g[0] == op.OK:
            assert op.predicted_peak(p, g[1]) <= M
            tot += 1
            opt += sum(cost[l] for l in g[1]) == sum(cost[l] for l in b[1])
    assert tot > 300
    # optimality is "parity unpinned" (near-optimal claim only)


@pytest.mark.parametrize("name", CFGS)
def test_budget_property_over_length_schedules(name):
    """c-H: simulated peak of the plan for x never exceeds M; INFEASIBLE iff LB > M."""
    cfg = wl.CONFIGS[name]
    Smax = cfg.max_seq
    szmax = om.sizes(cfg, cfg.n_seqs, Smax)
    C = szmax.C
    M = max(C + int(cfg.budget_frac * (om.no_ckpt_peak(szmax) - C)), om.lower_bound(szmax))
    samples = []
    for S in sorted({cfg.seq_lo, cfg.max_seq, (cfg.seq_lo + cfg.seq_hi) // 2}):
        S = wl.roundup(S, cfg.pad)
        c = om.collect_samples(om.sizes(cfg, cfg.n_seqs, S))
        c["x"] = cfg.n_seqs * S
        samples.append(c)
    est = oe.Estimator(samples)
    cache = op.PlanCache()
    prev_drops = -1
    for L_t in wl.length_schedule(cfg, 300):
        S = wl.roundup(L_t, cfg.pad)
        x = cfg.n_seqs * S
        st, dropped, pk = cache.get(x, lambda xx: op.plan(est.predict(xx), M))
        sz = om.sizes(cfg, cfg.n_seqs, S)
        assert st == op.OK
        assert om.peak(sz, dropped) <= M
        assert om.peak(sz, dropped) == pk        # exact predictions
    # plans grow with x (P:298 segments); below the no-drop threshold: no drops
    for S in range(cfg.pad, Smax + 1, cfg.pad):
        st, dropped, _ = op.plan(est.predict(cfg.n_seqs * S), M)
        assert len(dropped) >= prev_drops
        prev_drops = len(dropped)
        if om.no_ckpt_peak(om.sizes(cfg, cfg.n_seqs, S)) <= M:
            assert dropped == []
    # infeasible exactly when LB(x) > M
    tight = om.lower_bound(szmax) - 1
    st, _, _ = op.plan(est.predict(cfg.n_seqs * Smax), tight)
    assert st == op.INFEASIBLE


# ---------------------------------------------------------------------------
# sub-layer checkpoint units (DESIGN reading A30)
# ---------------------------------------------------------------------------

@pytest.mark.parametrize("name", POST_LN)
def test_units_event_model(name):
    """Unit event model: with nothing dropped it reaches the layer model's
    no-checkpoint peak (same push order); dropping every unit gives the unit
    collector's footprint; dropping only the FFN units of the first k layers
    lowers the peak by exactly k FFN-internal sizes (closed form, as for layers)."""
    cfg = wl.CONFIGS[name]
    L = cfg.n_layers
    for S in (cfg.seq_lo, cfg.max_seq):
        sz = om.sizes(cfg, cfg.n_seqs, S)
        P0 = om.no_ckpt_peak(sz)
        assert om.simulate_step_units(sz, []).peak == P0
        assert om.simulate_step_units(sz, [2 * L - 1]).peak == P0      # last unit saves nothing
        c = om.collect_samples_units(sz)
        assert om.simulate_step_units(sz, range(2 * L)).peak == c["peak"]
        i_att, i_ffn = sum(sz.internals[:5]), sum(sz.internals[6:])
        assert c["a"] == [i_att + sz.internals[5], i_ffn + sz.y] * L
        assert c["y"] == [sz.internals[5], sz.y] * L
        for k in range(L):
            # FFN units of layers 0..k-1 dropped: the layer-l backward event loses k FFN internals
            assert om.simulate_step_units(sz, [2 * j + 1 for j in range(k)]).peak == P0 - k * i_ffn


@pytest.mark.parametrize("name", CFGS)
def test_units_predicted_peak_formula(name):
    """The planner's position-aware peak over the 2L-unit collected series is
    exactly the unit event simulator's peak, for random unit plans."""
    cfg = wl.CONFIGS[name]
    rng = random.Random(21)
    for S in (cfg.seq_lo, cfg.max_seq):
        sz = om.sizes(cfg, cfg.n_seqs, S)
        c = om.collect_samples_units(sz)
        for _ in range(40):
            plan = rng.sample(range(2 * cfg.n_layers), rng.randint(0, 2 * cfg.n_layers))
            assert op.predicted_peak(c, plan) == om.simulate_step_units(sz, plan).peak


@pytest.mark.parametrize("name", CFGS)
def test_units_planners_feasible_and_exact(name):
    """Algorithm 1 on the unit series (heterogeneous: attention / FFN units
    alternate) returns a plan within the budget whenever one exists; the exact
    planner equals brute force (fewest units, then lowest peak, then lexicographic)."""
    cfg = wl.CONFIGS[name]
    L = cfg.n_layers
    sz = om.sizes(cfg, cfg.n_seqs, cfg.max_seq)
    c = om.collect_samples_units(sz)
    lo, hi = op.predicted_peak(c, range(2 * L)), op.predicted_peak(c, [])
    rng = random.Random(22)
    for _ in range(30 if 2 * L <= 12 else 6):
        M = rng.randint(lo - 1000, hi + 1000)
        g = op.plan(c, M)
        if g[0] == op.OK:
            assert om.simulate_step_units(sz, g[1]).peak <= M
        else:
            assert lo > M
        if 2 * L <= 12:
            e = op.plan_exact(c, M)
            b = op.brute_force(c, M, [1.0] * (2 * L))
            assert e[0] == b[0] and (e[0] != op.OK or (e[1] == b[1] and e[2] == b[2]))
