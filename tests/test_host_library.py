"""The C-ABI library on CPU (host-only context, no kernel launches):

* loads and exports every symbol include/mimose.h declares
* the arena's allocation sequence == the oracle's event model, byte for byte
  (dry-run peaks, collector samples) for every config and random plans
* C++ estimator and Algorithm-1 planner == the oracle, bit for bit
* the whole sheltered -> responsive pipeline (collect, fit, plan, cache) ==
  the oracle pipeline on the same length schedule
"""
import os
import random
import re

import numpy as np
import pytest

from oracle import estimator as oe
from oracle import memsim as om
from oracle import planner as op
from paper_conf_ipps_liaolysshfyctzlq23_b200 import binding as mb
from paper_conf_ipps_liaolysshfyctzlq23_b200 import workload as wl

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CFGS = ["toy", "bert-base", "bert-large", "roberta-large", "gpt2-medium"]
POST_LN = ["toy", "bert-base", "bert-large", "roberta-large"]


def test_exports_every_header_symbol():
    hdr = open(os.path.join(ROOT, "include", "mimose.h")).read()
    names = set(re.findall(r"\b(mimose_[a-z_0-9]+)\s*\(", hdr))
    assert len(names) >= 20
    for n in names:
        assert hasattr(mb._lib, n), n
    assert set(mb.EXPORTED) <= names


def budget_for(cfg):
    sz = om.sizes(cfg, cfg.n_seqs, cfg.max_seq)
    C = sz.C
    return max(C + int(cfg.budget_frac * (om.no_ckpt_peak(sz) - C)), om.lower_bound(sz))


@pytest.mark.parametrize("name", CFGS)
def test_dry_run_matches_event_model(name):
    cfg = wl.CONFIGS[name]
    ctx = mb.Mimose(cfg, budget_for(cfg))
    assert ctx.stats()["persistent_bytes"] == om.sizes(cfg, cfg.n_seqs, cfg.max_seq).C
    rng = random.Random(5)
    for S in sorted({cfg.pad, cfg.seq_lo, cfg.max_seq, wl.roundup((cfg.seq_lo + cfg.seq_hi) // 2, cfg.pad)}):
        sz = om.sizes(cfg, cfg.n_seqs, S)
        for _ in range(6):
            plan = rng.sample(range(cfg.n_layers), rng.randint(0, cfg.n_layers))
            assert ctx.dry_run(cfg.n_seqs, S, plan) == om.peak(sz, plan)
        got = ctx.dry_collect(cfg.n_seqs, S)
        want = om.collect_samples(sz)
        for k in ("C", "E", "Hd", "Th", "Tb", "Te", "a", "y"):
            assert got[k] == want[k], (k, S)


@pytest.mark.parametrize("name", CFGS)
def test_predicted_peak_and_planner_match_oracle(name):
    cfg = wl.CONFIGS[name]
    M = budget_for(cfg)
    rng = random.Random(6)
    for S in range(cfg.pad, cfg.max_seq + 1, max(cfg.pad, cfg.max_seq // 12)):
        p = om.collect_samples(om.sizes(cfg, cfg.n_seqs, S))
        for _ in range(3):
            plan = rng.sample(range(cfg.n_layers), rng.randint(0, cfg.n_layers))
            assert mb.predicted_peak(p, plan) == op.predicted_peak(p, plan)
        for budget in (M, M - 10**6, om.lower_bound(om.sizes(cfg, cfg.n_seqs, S)) - 1):
            st, dropped, pk = mb.plan_series(p, budget)
            ost, odropped, opk = op.plan(p, budget)
            assert (st == mb.OK) == (ost == op.OK)
            assert dropped == odropped and pk == opk


def test_planner_matches_oracle_on_random_stacks():
    rng = random.Random(8)
    for it in range(1500):
        L = rng.randint(1, 12)
        hom = it % 2 == 0
        ys = [rng.randint(1, 50)] * L if hom else [rng.randint(1, 50) for _ in range(L)]
        if hom:
            a = [ys[0] + rng.randint(1, 200)] * L
        else:
            a = [ys[l] + rng.randint(1, 200) for l in range(L)]
        p = dict(C=rng.randint(0, 1000), E=rng.randint(1, 100), a=a, y=ys, Hd=rng.randint(0, 20),
                 Th=rng.randint(1, 100), Tb=rng.randint(50, 400), Te=rng.randint(1, 300))
        lo, hi = op.predicted_peak(p, range(L)), op.predicted_peak(p, [])
        M = rng.randint(lo - 5, hi + 5)
        st, dropped, pk = mb.plan_series(p, M)
        ost, odropped, opk = op.plan(p, M)
        assert (st == mb.OK) == (ost == op.OK)
        assert dropped == odropped and pk == opk


def test_fit_predict_matches_oracle():
    rng = np.random.default_rng(2)
    for _ in range(200):
        xs = sorted(set(int(v) for v in rng.integers(100, 40000, size=12)))[:10]
        c0, c1, c2 = int(rng.integers(0, 10**9)), int(rng.integers(0, 10**6)), int(rng.integers(0, 1000))
        ys = [c0 + c1 * x + c2 * x * x for x in xs]
        xe = list(rng.integers(1, 60000, size=20))
        got = mb.fit_predict(xs, ys, xe)
        q = oe.Quadratic(xs, ys)
        assert got == [q.predict(int(x)) for x in xe]
        assert got == [c0 + c1 * int(x) + c2 * int(x) ** 2 for x in xe]
    # degree fallbacks and the residual margin
    assert mb.fit_predict([100, 100, 200], [5, 5, 9], [300]) == [13]
    assert mb.fit_predict([100, 100], [5, 5], [999]) == [5]
    xs, ys = [1, 2, 3, 4], [0, 10, 0, 10]
    assert mb.fit_predict(xs, ys, xs) == [oe.Quadratic(xs, ys).predict(x) for x in xs]


@pytest.mark.parametrize("name", CFGS)
def test_sheltered_to_responsive_pipeline_matches_oracle(name):
    cfg = wl.CONFIGS[name]
    M = budget_for(cfg)
    ctx = mb.Mimose(cfg, M)
    sched = wl.length_schedule(cfg, 200)
    samples, seen, i = [], set(), 0
    while ctx.phase == mb.PHASE_SHELTERED:
        b = wl.make_batch(cfg, sched[i], seed=i)
        ctx.collect(ctx.host_batch(b))
        ctx.backward()
        x = b.input_size
        if x not in seen:
            seen.add(x)
            s = om.collect_samples(om.sizes(cfg, cfg.n_seqs, b.seq_len))
            s["x"] = x
            samples.append(s)
        i += 1
    st = ctx.stats()
    assert st["n_samples"] == len(samples) and st["collect_steps"] == i
    assert i >= 10 and len(samples) >= 3
    for j, s in enumerate(samples):
        got = ctx.sample(j)
        for k in ("x", "C", "E", "Hd", "Th", "Tb", "Te", "a", "y"):
            assert got[k] == s[k]
    est = oe.Estimator(samples)
    cache = op.PlanCache()
    for L_t in sched[i:]:
        S = wl.roundup(L_t, cfg.pad)
        x = cfg.n_seqs * S
        p = ctx.plan(x)
        ost, odropped, opk = cache.get(x, lambda xx: op.plan(est.predict(xx), M))
        assert p.status == mb.OK and ost == op.OK
        assert p.dropped == odropped and p.predicted_peak == opk
        assert ctx.dry_run(cfg.n_seqs, S, p.dropped) == om.peak(om.sizes(cfg, cfg.n_seqs, S), p.dropped) <= M
    st = ctx.stats()
    assert st["plan_cache_hits"] == cache.hits and st["plan_cache_misses"] == cache.misses


def test_call_order_and_budget_errors():
    cfg = wl.CONFIGS["toy"]
    M = budget_for(cfg)
    ctx = mb.Mimose(cfg, M)
    with pytest.raises(mb.MimoseError) as e:
        ctx.plan(64)
    assert e.value.status == mb.E_NOT_READY
    with pytest.raises(mb.MimoseError) as e:
        ctx.backward()
    assert e.value.status == mb.E_STATE
    b = wl.make_batch(cfg, 32, seed=1)
    # no-checkpoint forward of the largest input breaks the 50% budget -> violation, nothing launched
    with pytest.raises(mb.MimoseError) as e:
        ctx.forward(ctx.host_batch(b))
    assert e.value.status == mb.E_BUDGET
    assert ctx.stats()["violations"] == 1
    with pytest.raises(mb.MimoseError) as e:
        mb.Mimose(cfg, om.sizes(cfg, 2, 32).C - 1)
    assert e.value.status == mb.E_INFEASIBLE


def _random_series(rng, L, hom):
    ys = [rng.randint(1, 50)] * L if hom else [rng.randint(1, 50) for _ in range(L)]
    a = [ys[0] + rng.randint(1, 200)] * L if hom else [ys[l] + rng.randint(1, 200) for l in range(L)]
    return dict(C=rng.randint(0, 1000), E=rng.randint(1, 100), a=a, y=ys, Hd=rng.randint(0, 20),
                Th=rng.randint(1, 100), Tb=rng.randint(50, 400), Te=rng.randint(1, 300))


def test_exact_planner_matches_brute_force():
    """Reading A29: the library's exact planner (mimose_set_planner kind 1) equals
    the oracle's brute force over all drop sets (fewest layers, then lowest
    peak, then lexicographically smallest), and never recomputes more layers
    than Algorithm 1; on homogeneous stacks the two coincide."""
    rng = random.Random(29)
    fewer = 0
    for it in range(800):
        L = rng.randint(1, 11)
        hom = it % 2 == 0
        p = _random_series(rng, L, hom)
        lo, hi = op.predicted_peak(p, range(L)), op.predicted_peak(p, [])
        M = rng.randint(lo - 5, hi + 5)
        st, dropped, pk = mb.plan_series(p, M, planner=mb.PLANNER_EXACT)
        ost, odropped, opk = op.plan_exact(p, M)
        assert (st == mb.OK) == (ost == op.OK)
        if ost == op.OK:
            assert dropped == odropped and pk == opk <= M
            gst, gdropped, gpk = mb.plan_series(p, M)
            assert gst == mb.OK and len(dropped) <= len(gdropped)
            if hom:
                assert dropped == gdropped and pk == gpk
            fewer += len(dropped) < len(gdropped)
    assert fewer > 0        # heterogeneous stacks where the exact plan recomputes less


@pytest.mark.parametrize("name", CFGS)
def test_exact_planner_on_config_series(name):
    """24-layer series of the real configs: feasible whenever greedy is, never
    more layers, within the budget, and fast enough for a cache miss."""
    import time
    cfg = wl.CONFIGS[name]
    M = budget_for(cfg)
    worst = 0.0
    for S in range(cfg.pad, cfg.max_seq + 1, max(cfg.pad, cfg.max_seq // 8)):
        p = om.collect_samples(om.sizes(cfg, cfg.n_seqs, S))
        t0 = time.perf_counter()
        st, dropped, pk = mb.plan_series(p, M, planner=mb.PLANNER_EXACT)
        worst = max(worst, time.perf_counter() - t0)
        gst, gdropped, gpk = mb.plan_series(p, M)
        assert (st == mb.OK) == (gst == mb.OK)
        if st == mb.OK:
            assert pk <= M and pk == op.predicted_peak(p, dropped) and len(dropped) <= len(gdropped)
    assert worst < 0.5, worst


def test_time_weighted_planner_matches_brute_force():
    """Reading A31: the library's cost-weighted exact planner (kind 2, a dynamic
    program with dominance pruning) equals the oracle's brute force (least
    total integer cost, then lowest peak, then lexicographic) bit for bit, on
    homogeneous and heterogeneous stacks with random costs, including ties."""
    rng = random.Random(31)
    n_ok = 0
    for it in range(1200):
        L = rng.randint(1, 11)
        p = _random_series(rng, L, it % 2 == 0)
        cost = ([rng.randint(1, 4) for _ in range(L)] if it % 3 == 0 else
                [rng.randint(0, 10 ** 6) for _ in range(L)])
        lo, hi = op.predicted_peak(p, range(L)), op.predicted_peak(p, [])
        M = rng.randint(lo - 5, hi + 5)
        st, dropped, pk = mb.plan_series_cost(p, cost, M)
        ost, odropped, opk = op.plan_exact_cost(p, M, cost)
        assert (st == mb.OK) == (ost == op.OK), (p, cost, M)
        if ost == op.OK:
            assert dropped == odropped and pk == opk <= M, (p, cost, M)
            n_ok += 1
    assert n_ok > 500


@pytest.mark.parametrize("name", CFGS)
def test_time_weighted_planner_scales_to_units(name):
    """48-unit series (H = 1024 configs at granularity 1) with attention / FFN
    recompute costs from the FLOP model: feasible whenever a plan exists, within
    the budget, never costlier than the unit-count exact plan, and fast."""
    import time
    cfg = wl.CONFIGS[name]
    M = budget_for(cfg)
    H, F = cfg.hidden, cfg.ffn
    worst = 0.0
    for S in range(cfg.pad, cfg.max_seq + 1, max(cfg.pad, cfg.max_seq // 6)):
        p = om.collect_samples_units(om.sizes(cfg, cfg.n_seqs, S))
        T = cfg.n_seqs * S
        cost = [2 * T * 4 * H * H + 4 * cfg.n_seqs * S * S * H, 2 * T * 2 * H * F] * cfg.n_layers
        cost = [c // 10 ** 6 + 1 for c in cost]
        t0 = time.perf_counter()
        st, dropped, pk = mb.plan_series_cost(p, cost, M)
        worst = max(worst, time.perf_counter() - t0)
        est, edropped, _ = mb.plan_series(p, M, planner=mb.PLANNER_EXACT)
        assert (st == mb.OK) == (est == mb.OK)
        if st == mb.OK:
            assert pk <= M and pk == op.predicted_peak(p, dropped)
            assert sum(cost[u] for u in dropped) <= sum(cost[u] for u in edropped)
    assert worst < 0.5, worst


# ---------------------------------------------------------------------------
# sub-layer checkpoint units (granularity=1, DESIGN reading A30)
# ---------------------------------------------------------------------------
UNIT_CFGS = ["toy", "bert-base", "bert-large", "roberta-large", "gpt2-medium"]


@pytest.mark.parametrize("name", UNIT_CFGS)
def test_units_dry_run_and_collector_match_event_model(name):
    """Host-only ctx at granularity 1: the arena's dry-run peak of random unit
    plans and the unit collector's samples equal oracle/memsim's unit model."""
    cfg = wl.CONFIGS[name]
    ctx = mb.Mimose(cfg, budget_for(cfg), granularity=1)
    assert ctx.n_units == 2 * cfg.n_layers
    rng = random.Random(15)
    for S in sorted({cfg.pad, cfg.seq_lo, cfg.max_seq}):
        sz = om.sizes(cfg, cfg.n_seqs, S)
        for _ in range(6):
            plan = rng.sample(range(2 * cfg.n_layers), rng.randint(0, 2 * cfg.n_layers))
            assert ctx.dry_run(cfg.n_seqs, S, plan) == om.simulate_step_units(sz, plan).peak
        got = ctx.dry_collect(cfg.n_seqs, S)
        want = om.collect_samples_units(sz)
        for k in ("C", "E", "Hd", "Th", "Tb", "Te", "a", "y"):
            assert got[k] == want[k], (k, S)


@pytest.mark.parametrize("name,planner", [(n, "greedy") for n in UNIT_CFGS] + [("toy", "exact")])
def test_units_pipeline_matches_oracle(name, planner):
    """Sheltered phase -> estimator -> Algorithm 1 (or the exact planner, whose
    oracle is brute force: toy only) over the 2L units: every plan equals the
    oracle's, and its simulated peak is within the budget."""
    cfg = wl.CONFIGS[name]
    M = budget_for(cfg)
    ctx = mb.Mimose(cfg, M, granularity=1)
    if planner == "exact":
        ctx.set_planner(1)
    sched = wl.length_schedule(cfg, 120)
    samples, seen, i = [], set(), 0
    while ctx.phase == mb.PHASE_SHELTERED:
        b = wl.make_batch(cfg, sched[i], seed=i)
        ctx.collect(ctx.host_batch(b))
        ctx.backward()
        if b.input_size not in seen:
            seen.add(b.input_size)
            s = om.collect_samples_units(om.sizes(cfg, cfg.n_seqs, b.seq_len))
            s["x"] = b.input_size
            samples.append(s)
        i += 1
    for j, s in enumerate(samples):
        got = ctx.sample(j)
        for k in ("x", "C", "E", "Hd", "Th", "Tb", "Te", "a", "y"):
            assert got[k] == s[k]
    est = oe.Estimator(samples)
    fn = op.plan if planner == "greedy" else op.plan_exact
    for L_t in sched[i:i + 40]:
        S = wl.roundup(L_t, cfg.pad)
        x = cfg.n_seqs * S
        p = ctx.plan(x)
        ost, odropped, opk = fn(est.predict(x), M)
        assert p.status == mb.OK and ost == op.OK
        assert p.dropped == list(odropped) and p.predicted_peak == opk
        assert ctx.dry_run(cfg.n_seqs, S, p.dropped) == om.simulate_step_units(
            om.sizes(cfg, cfg.n_seqs, S), p.dropped).peak <= M


def test_units_config_validation():
    """granularity is 0 or 1, and 2L units must fit the 64-bit drop mask."""
    with pytest.raises(mb.MimoseError):
        mb.Mimose(wl.CONFIGS["toy"], 1 << 40, granularity=2)
    with pytest.raises(mb.MimoseError):
        mb.Mimose(wl.small_config("bert-base", n_layers=33), 1 << 40, granularity=1)
