"""ORACLE (test infrastructure only): Mimose's greedy scheduler (Algorithm 1,
PAPER.md P:186-213, prose P:177-179), the position-aware predicted peak used
to verify a plan, the plan cache, and a brute-force reference.

Readings (DESIGN.md register, numbered as SURVEY §8(c)-R):
  A1/A2  restore the lost minus signs: excess = sum est - M ; excess -= est[l]
  A4     est_mem[l] = droppable bytes d_l = a_l - y_l (collector pass1 - pass2)
  A5     stable sort, ties -> earlier layer
  A6     bucket test 10*est[j] > 9*est[head] (strict, integers)
  A7/A9  a bucket's "top" = its earliest layer; line 17 takes the earliest
         layer of the first (largest) bucket
  A8     line 19 takes the candidate bucket with the SMALLEST max above the
         excess ("nearest to the excess memory")
  A10    loop while excess > 0
  A11    no layers left -> INFEASIBLE
  A12    the last layer is not a candidate; it is tried only as a
         last resort before INFEASIBLE
  A13    when the linear accounting says excess <= 0, re-check with the
         position-aware predicted peak P(L',x) and continue if still over
  A31    the time-weighted exact planner (the Knapsack of P:179): minimum
         total integer recompute cost, then peak, then lexicographic
         = brute_force(cost) (plan_exact_cost)
  A29    the exact alternative planner ("a flexible interface for ...
         other scheduling algorithms, such as the Knapsack optimization"):
         fewest recomputed layers (unit cost: homogeneous encoder layers)
         with predicted_peak <= M - reserve, then the lowest peak, then the
         lexicographically smallest sorted layer list = brute_force(cost=1)
All byte arithmetic is in Python integers.

Pinned by: hand traces (tests/golden/alg1_traces.txt), brute force over all
subsets on <=10-layer stacks evaluated with the event simulator
(brute_force_sim; tests/test_oracle_pins.py), budget property tests.  Optimality on
heterogeneous stacks is "parity unpinned" (the paper claims near-optimal only).
"""
from __future__ import annotations

import itertools
from typing import Dict, List, Optional, Sequence, Tuple

OK = "ok"
INFEASIBLE = "infeasible"


def predicted_peak(p: Dict, dropped: Sequence[int]) -> int:
    """Peak of the arena event model (memsim.simulate_step) evaluated on
    per-series sizes p = {C, E, a[l], y[l], Hd, Th, Tb, Te}."""
    drop = set(dropped)
    L = len(p["a"])
    base = p["C"] + p["E"]
    pk = base + p["Te"]
    S = 0
    prefix = []
    for l in range(L):
        prefix.append(S)
        pk = max(pk, base + S + p["a"][l])                     # forward of layer l
        S += p["y"][l] if l in drop else p["a"][l]
    pk = max(pk, base + S + p["Hd"] + p["Th"])                 # head backward
    for l in range(L):
        pk = max(pk, base + prefix[l] + (p["a"][l] - p["y"][l]) + p["Tb"])
    return pk


def make_buckets(est: Sequence[int], cands: Sequence[int]) -> List[List[int]]:
    """Alg. 1 lines 2-12."""
    order = sorted(cands, key=lambda l: (-est[l], l))          # line 3 (A5)
    buckets = []
    i = 0
    while i < len(order):                                      # line 4
        head = order[i]
        bucket = [head]
        i += 1
        while i < len(order) and 10 * est[order[i]] > 9 * est[head]:   # line 8 (A6)
            bucket.append(order[i])
            i += 1
        buckets.append(sorted(bucket))                         # line 11 (A7)
    return buckets


def greedy_select(est: Sequence[int], buckets: List[List[int]], excess: int,
                  chosen: List[int]) -> Tuple[int, bool]:
    """Alg. 1 lines 14-21 on mutable buckets; returns (excess, exhausted)."""
    while excess > 0:                                          # line 14 (A10)
        if not buckets:
            return excess, True
        cands = [b for b in buckets if max(est[l] for l in b) > excess]   # line 15
        if not cands:
            b = buckets[0]                                     # line 17 (A9)
        else:
            b = min(cands, key=lambda bb: max(est[l] for l in bb))        # line 19 (A8)
        l = b[0]
        chosen.append(l)                                       # line 20
        b.remove(l)
        if not b:
            buckets.remove(b)
        excess -= est[l]                                       # line 21 (A2)
    return excess, False


def greedy_core(est: Sequence[int], excess: int, candidates: Optional[Sequence[int]] = None):
    """Algorithm 1 alone, given est and the initial excess (hand traces)."""
    cands = list(range(len(est))) if candidates is None else list(candidates)
    buckets = make_buckets(est, cands)
    chosen: List[int] = []
    exc, exhausted = greedy_select(est, buckets, excess, chosen)
    return (INFEASIBLE if exhausted else OK), sorted(chosen), [list(b) for b in make_buckets(est, cands)]


def plan(p: Dict, budget: int, reserve: int = 0):
    """Full planner: Alg. 1 + A12 + A13.  Returns (status, dropped, predicted_peak)."""
    L = len(p["a"])
    limit = budget - reserve
    est = [p["a"][l] - p["y"][l] for l in range(L)]            # A4
    chosen: List[int] = []
    pk = predicted_peak(p, chosen)
    excess = pk - limit                                        # line 13 (A1)
    buckets = make_buckets(est, range(L - 1))                  # A12
    while True:
        excess, exhausted = greedy_select(est, buckets, excess, chosen)
        if exhausted:
            break
        pk = predicted_peak(p, chosen)                         # A13 verify
        excess = pk - limit
        if excess <= 0:
            return OK, sorted(chosen), pk
    if L - 1 not in chosen:                                    # A12 last resort
        chosen.append(L - 1)
        pk = predicted_peak(p, chosen)
        if pk <= limit:
            return OK, sorted(chosen), pk
    return INFEASIBLE, sorted(chosen), predicted_peak(p, chosen)


class PlanCache:
    """Plans indexed by input size ("uses the input tensor size as the
    indexing key"); the key is x = B*S_pad, S_pad already bucketed (A16)."""

    def __init__(self):
        self.cache: Dict[int, Tuple] = {}
        self.hits = 0
        self.misses = 0

    def get(self, x: int, make):
        if x in self.cache:
            self.hits += 1
            return self.cache[x]
        self.misses += 1
        v = make(x)
        self.cache[x] = v
        return v


def brute_force(p: Dict, budget: int, cost: Sequence[float], reserve: int = 0):
    """All 2^L subsets: feasible with minimum sum(cost), then minimum peak,
    then lexicographically smallest.  Returns (status, dropped, peak)."""
    L = len(p["a"])
    best = None
    for k in range(L + 1):
        for sub in itertools.combinations(range(L), k):
            pk = predicted_peak(p, sub)
            if pk > budget - reserve:
                continue
            key = (sum(cost[l] for l in sub), pk, sub)
            if best is None or key < best:
                best = key
    if best is None:
        return INFEASIBLE, None, None
    return OK, list(best[2]), best[1]


def brute_force_sim(peak_of, n_units: int, budget: int, cost: Sequence[float], reserve: int = 0):
    """SURVEY c-G's brute-force pin: all 2^n drop sets evaluated with the EVENT
    SIMULATOR (``peak_of(dropped)``, e.g. memsim.simulate_step on the true
    Sizes), not with the planner's own predicted-peak formula.  Feasible with
    minimum sum(cost), then minimum peak, then lexicographically smallest."""
    best = None
    for k in range(n_units + 1):
        for sub in itertools.combinations(range(n_units), k):
            pk = peak_of(sub)
            if pk > budget - reserve:
                continue
            key = (sum(cost[l] for l in sub), pk, sub)
            if best is None or key < best:
                best = key
    if best is None:
        return INFEASIBLE, None, None
    return OK, list(best[2]), best[1]


def plan_exact(p: Dict, budget: int, reserve: int = 0):
    """Reading A29: the exact planner is, by definition, the brute-force
    minimum over all 2^L drop sets with unit recompute cost (small L only).
    An infeasible budget returns (INFEASIBLE, all layers, their peak)."""
    L = len(p["a"])
    st, dropped, pk = brute_force(p, budget, [1] * L, reserve)
    if st != OK:
        return INFEASIBLE, list(range(L)), predicted_peak(p, range(L))
    return OK, dropped, pk


def plan_exact_cost(p: Dict, budget: int, cost: Sequence[int], reserve: int = 0):
    """Reading A31 ("Knapsack"): the time-weighted exact planner is, by
    definition, the brute-force minimum over all 2^L drop sets of the total
    integer recompute cost (each cost clamped to >= 1), then the lowest peak,
    then the lexicographically smallest sorted layer list.  Infeasible ->
    (INFEASIBLE, all layers, their peak)."""
    L = len(p["a"])
    st, dropped, pk = brute_force(p, budget, [max(1, int(c)) for c in cost], reserve)
    if st != OK:
        return INFEASIBLE, list(range(L)), predicted_peak(p, range(L))
    return OK, dropped, pk
