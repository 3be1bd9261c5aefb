"""Encoder-decoder memory model, 2-D estimator and planning (
reading A32), oracle side (CPU):

* the planner's position-aware peak over the Le + Ld unit series equals the
  encoder-decoder event simulator for random plans (exactness of A13's model);
* closed forms: the collector's footprint is the all-dropped peak; P(empty)
  and LB; peak monotone in each of the two input sizes;
* the bivariate quadratic estimator recovers integer bivariate polynomials
  exactly (incl. extrapolation) and falls back to degree 1 / 0 with too few
  distinct key pairs; on the collected series of the model it predicts every
  size exactly;
* Algorithm 1 on the estimator's predictions equals brute force over the
  simulator on a 3 + 3 layer model, and keeps every step of a 2-D length
  schedule within the budget (INFEASIBLE exactly when LB > M).
"""
import random

import numpy as np
import pytest

from oracle import estimator as oe
from oracle import memsim as om
from oracle import planner as op
from paper_conf_ipps_liaolysshfyctzlq23_b200 import workload as wl

CFG = wl.CONFIGS["t5-base"]


def pairs(cfg, n, seed):
    rng = np.random.default_rng(seed)
    out = []
    for _ in range(n):
        b = wl.make_batch(cfg, int(rng.integers(cfg.seq_lo, cfg.seq_hi + 1)), seed=int(rng.integers(1 << 30)))
        out.append((b.seq_len, b.dec_len))
    return out


def test_predicted_peak_equals_simulator():
    rng = random.Random(3)
    n = CFG.n_layers + CFG.n_dec_layers
    for Ss, St in [(24, 24), (64, 72), (128, 104), (40, 128), (128, 16)]:
        sz = om.sizes_encdec(CFG, CFG.n_seqs, Ss, St)
        c = om.collect_samples_encdec(sz)
        assert c["peak"] == om.simulate_step_encdec(sz, range(n)).peak
        for _ in range(100):
            plan = rng.sample(range(n), rng.randint(0, n))
            assert op.predicted_peak(c, plan) == om.simulate_step_encdec(sz, plan).peak


def test_monotone_in_both_sizes():
    rng = random.Random(4)
    n = CFG.n_layers + CFG.n_dec_layers
    for _ in range(5):
        plan = rng.sample(range(n), rng.randint(0, n))
        for St in (16, 64, 128):
            prev = 0
            for Ss in range(8, 129, 8):
                pk = om.simulate_step_encdec(om.sizes_encdec(CFG, CFG.n_seqs, Ss, St), plan).peak
                assert pk >= prev
                prev = pk
        for Ss in (16, 128):
            prev = 0
            for St in range(8, 129, 8):
                pk = om.simulate_step_encdec(om.sizes_encdec(CFG, CFG.n_seqs, Ss, St), plan).peak
                assert pk >= prev
                prev = pk


def test_quadratic2d_exact_and_fallbacks():
    rng = np.random.default_rng(7)
    pts = [(8 * a, 8 * b) for a, b in rng.integers(2, 130, size=(12, 2))]
    for _ in range(30):
        c = [int(v) for v in rng.integers(0, 10 ** 9, 6)]
        c[1] //= 1000; c[2] //= 1000; c[3] //= 10 ** 6; c[4] //= 10 ** 6; c[5] //= 10 ** 6
        f = lambda x, t: c[0] + c[1] * x + c[2] * t + c[3] * x * x + c[4] * x * t + c[5] * t * t
        q = oe.Quadratic2D([p[0] for p in pts], [p[1] for p in pts], [f(*p) for p in pts])
        assert q.degree == 2 and q.margin == 0
        for x in (16, 512, 1040, 1600):
            for t in (16, 400, 1040, 1500):
                assert q.predict(x, t) == f(x, t)
    # too few distinct pairs: degree 1 (3 non-collinear), constant (1 pair)
    q = oe.Quadratic2D([100, 200, 100, 100], [100, 100, 300, 100], [5, 7, 11, 5])
    assert q.degree == 1 and q.predict(300, 300) == 5 + 2 * 2 + 3 * 2
    q = oe.Quadratic2D([100, 100], [50, 50], [9, 9])
    assert q.degree == 0 and q.predict(1, 1) == 9
    # collinear pairs (t = x) cannot separate s from t: degree 0
    q = oe.Quadratic2D([10, 20, 30], [10, 20, 30], [1, 2, 3])
    assert q.degree == 0 and all(q.predict(x, x) >= y for x, y in ((10, 1), (20, 2), (30, 3)))


def test_estimator2d_exact_on_collected_series():
    samples = []
    for Ss, St in pairs(CFG, 10, 11):
        c = om.collect_samples_encdec(om.sizes_encdec(CFG, CFG.n_seqs, Ss, St))
        c["x"], c["xt"] = CFG.n_seqs * Ss, CFG.n_seqs * St
        samples.append(c)
    est = oe.Estimator2D(samples)
    for Ss in range(8, 129, 24):
        for St in range(8, 129, 24):
            truth = om.collect_samples_encdec(om.sizes_encdec(CFG, CFG.n_seqs, Ss, St))
            pred = est.predict(CFG.n_seqs * Ss, CFG.n_seqs * St)
            for k in ("E", "Hd", "Th", "Tb", "Te", "a", "y"):
                assert pred[k] == truth[k], (k, Ss, St)


def budget(cfg):
    sz = om.sizes_encdec(cfg, cfg.n_seqs, cfg.max_seq, cfg.max_seq)
    n = cfg.n_layers + cfg.n_dec_layers
    P0, LB = om.simulate_step_encdec(sz, []).peak, om.simulate_step_encdec(sz, range(n)).peak
    return max(sz.C + int(cfg.budget_frac * (P0 - sz.C)), LB)


def test_greedy_equals_simulator_brute_force_small():
    cfg = wl.small_config("t5-base", n_layers=3, n_dec_layers=3, n_seqs=8)
    n = 6
    rng = random.Random(5)
    n_ok = 0
    for Ss, St in [(128, 128), (64, 96), (32, 24)]:
        sz = om.sizes_encdec(cfg, cfg.n_seqs, Ss, St)
        c = om.collect_samples_encdec(sz)
        lo, hi = om.simulate_step_encdec(sz, range(n)).peak, om.simulate_step_encdec(sz, []).peak
        memo = {}

        def pk(D):
            D = tuple(sorted(D))
            if D not in memo:
                memo[D] = om.simulate_step_encdec(sz, D).peak
            return memo[D]

        for M in [lo - 1, lo, hi] + [rng.randint(lo, hi) for _ in range(6)]:
            g = op.plan(c, M)
            b = op.brute_force_sim(pk, n, M, [1.0] * n)
            assert g[0] == b[0]
            if g[0] == op.OK:
                assert pk(g[1]) <= M
                e = op.plan_exact(c, M)
                assert (e[1], e[2]) == (b[1], b[2])
                n_ok += 1
    assert n_ok >= 10


def test_budget_property_over_a_2d_schedule():
    M = budget(CFG)
    samples = []
    for Ss, St in pairs(CFG, 10, 12):
        c = om.collect_samples_encdec(om.sizes_encdec(CFG, CFG.n_seqs, Ss, St))
        c["x"], c["xt"] = CFG.n_seqs * Ss, CFG.n_seqs * St
        samples.append(c)
    est = oe.Estimator2D(samples)
    n_drop = 0
    for Ss, St in pairs(CFG, 200, 13):
        st, dropped, pk = op.plan(est.predict(CFG.n_seqs * Ss, CFG.n_seqs * St), M)
        sz = om.sizes_encdec(CFG, CFG.n_seqs, Ss, St)
        assert st == op.OK and om.simulate_step_encdec(sz, dropped).peak == pk <= M
        n_drop += len(dropped) > 0
    assert n_drop > 0
    szmax = om.sizes_encdec(CFG, CFG.n_seqs, CFG.max_seq, CFG.max_seq)
    tight = om.simulate_step_encdec(szmax, range(24)).peak - 1
    st, _, _ = op.plan(est.predict(CFG.n_seqs * CFG.max_seq, CFG.n_seqs * CFG.max_seq), tight)
    assert st == op.INFEASIBLE


# ---------------------------------------------------------------- library --

def test_library_accounting_matches_oracle():
    from paper_conf_ipps_liaolysshfyctzlq23_b200 import binding as mb
    ctx = mb.Mimose(CFG, budget(CFG))
    assert ctx.n_params == wl.n_params(CFG) and ctx.n_units == 24
    assert ctx.stats()["persistent_bytes"] == om.persistent_bytes(CFG, CFG.n_seqs, CFG.max_seq)
    rng = random.Random(8)
    for Ss, St in [(24, 24), (64, 72), (128, 104), (40, 128), (128, 16)]:
        sz = om.sizes_encdec(CFG, CFG.n_seqs, Ss, St)
        for _ in range(10):
            plan = rng.sample(range(24), rng.randint(0, 24))
            assert ctx.dry_run(CFG.n_seqs, Ss, plan, dec_len=St) == om.simulate_step_encdec(sz, plan).peak
        got, want = ctx.dry_collect(CFG.n_seqs, Ss, dec_len=St), om.collect_samples_encdec(sz)
        assert got["xt"] == CFG.n_seqs * St
        for k in ("C", "E", "Hd", "Th", "Tb", "Te", "a", "y"):
            assert got[k] == want[k], k


def test_library_pipeline_matches_oracle():
    """Sheltered phase on 2-D keys -> bivariate fit -> mimose_plan2 (Algorithm
    1): every plan equals the oracle planner on the oracle's Estimator2D, within
    the budget.  (The exact planners' oracle is brute force: 3 + 3 layers above.)"""
    from paper_conf_ipps_liaolysshfyctzlq23_b200 import binding as mb
    M = budget(CFG)
    ctx = mb.Mimose(CFG, M)
    rng = np.random.default_rng(21)
    samples, seen = [], set()
    i = 0
    while ctx.phase == mb.PHASE_SHELTERED:
        b = wl.make_batch(CFG, int(rng.integers(CFG.seq_lo, CFG.seq_hi + 1)), seed=i)
        ctx.collect(ctx.host_batch(b))
        ctx.backward()
        key = b.input_size2
        if key not in seen:
            seen.add(key)
            s = om.collect_samples_encdec(om.sizes_encdec(CFG, CFG.n_seqs, b.seq_len, b.dec_len))
            s["x"], s["xt"] = key
            samples.append(s)
        i += 1
    assert len(samples) >= 6
    for j, s in enumerate(samples):
        got = ctx.sample(j)
        for k in ("x", "xt", "C", "E", "Hd", "Th", "Tb", "Te", "a", "y"):
            assert got[k] == s[k], k
    est = oe.Estimator2D(samples)
    fn = op.plan
    n_drop = 0
    for Ss, St in pairs(CFG, 60, 22):
        x, xt = CFG.n_seqs * Ss, CFG.n_seqs * St
        p = ctx.plan(x, xt)
        ost, od, opk = fn(est.predict(x, xt), M)
        assert p.status == mb.OK and ost == op.OK
        assert p.dropped == list(od) and p.predicted_peak == opk
        assert ctx.dry_run(CFG.n_seqs, Ss, p.dropped, dec_len=St) <= M
        n_drop += len(od) > 0
    assert n_drop > 0
    with pytest.raises(mb.MimoseError):
        ctx.plan(CFG.n_seqs * 64)                         # the 1-D call is refused
