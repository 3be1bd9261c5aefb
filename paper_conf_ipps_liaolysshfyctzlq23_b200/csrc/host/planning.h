// Host-side Mimose planning: lightning memory estimator (§IV-C,
// P:144-164; §VI-E) and the greedy scheduler (§IV-D, Algorithm 1
// P:186-213) with the readings of DESIGN.md (A1-A13, A18).  Pure C++, no CUDA.
#pragma once
#include <cstdint>
#include <unordered_map>
#include <vector>

namespace mimose {

// Quadratic least squares in t = x / x_ref (reading A18): normal equations,
// Gaussian elimination with partial pivoting, Horner evaluation, integer
// predictions rounded half-to-even plus a non-negative residual margin.
struct Poly {
  int degree = 0;
  double x_ref = 1.0;
  double coef[3] = {0, 0, 0};
  int64_t margin = 0;
  void fit(const std::vector<int64_t>& xs, const std::vector<int64_t>& ys, int max_degree);
  double eval(int64_t x) const;
  int64_t predict(int64_t x) const;
};

// Bivariate least squares for the 2-D key of an encoder-decoder (reading A32):
// features [1, s, t, s^2, s t, t^2] (degree 2), [1, s, t] (degree 1) or [1],
// s = x / x_ref, t = xt / t_ref; the highest degree whose design matrix has
// full rank on the distinct key pairs; normal equations with partial pivoting.
struct Poly2 {
  int degree = 0, nf = 1;
  double x_ref = 1.0, t_ref = 1.0;
  double coef[6] = {0, 0, 0, 0, 0, 0};
  int64_t margin = 0;
  void fit(const std::vector<int64_t>& xs, const std::vector<int64_t>& ts, const std::vector<int64_t>& ys,
           int max_degree);
  double eval(int64_t x, int64_t xt) const;
  int64_t predict(int64_t x, int64_t xt) const;
};

// Per-series sizes for one input size x (what the planner reasons about).
struct Series {
  int64_t C = 0, E = 0, Hd = 0, Th = 0, Tb = 0, Te = 0;
  std::vector<int64_t> a, y;   // per layer
};

// Position-aware peak of the arena event model (reading A13).
int64_t predicted_peak(const Series& s, uint64_t drop_mask);

struct PlanResult {
  bool feasible = false;
  uint64_t drop_mask = 0;
  int64_t peak = 0;
};
// Algorithm 1 (A1-A11) + last-layer exclusion (A12) + verify (A13).
PlanResult plan_greedy(const Series& s, int64_t budget, int64_t reserve, int bucket_num, int bucket_den);

// The exact alternative behind the same (M, x, L) -> L' interface ("a
// flexible interface ... such as the Knapsack optimization"): among all drop
// sets whose position-aware predicted peak is <= budget - reserve, the one with
// the fewest recomputed layers (unit recompute cost: the encoder layers are
// homogeneous), then the lowest peak, then the lexicographically smallest
// sorted layer list (reading A29): plan_exact_cost with every cost 1.
PlanResult plan_exact(const Series& s, int64_t budget, int64_t reserve);

// The recompute-time-weighted exact planner ("Knapsack", reading
// A31): among all feasible drop sets, the minimum total recompute cost
// sum cost[l] (integers, each >= 1), then the lowest peak, then the
// lexicographically smallest sorted layer list.  Three exact phases, each a
// forward dynamic program over the layers with the 2-D Pareto front of
// (stack bytes, cost): the least cost; the lowest peak among least-cost sets
// (binary search on the event limit); then the lexicographic choice layer by
// layer.  Milliseconds at 48 units.
PlanResult plan_exact_cost(const Series& s, const std::vector<int64_t>& cost, int64_t budget, int64_t reserve);
enum PlannerKind : int { PLANNER_GREEDY = 0, PLANNER_EXACT = 1, PLANNER_EXACT_TIME = 2 };

// One collected sheltered-iteration sample (arena deltas).
struct Sample {
  int64_t x = 0, xt = 0, C = 0, E = 0, Hd = 0, Th = 0, Tb = 0, Te = 0;
  std::vector<int64_t> a, y;
  std::vector<float> t_ms;
};

struct Estimator {
  bool fitted = false;
  int64_t C = 0;
  std::vector<Poly> fa, fy;
  Poly fE, fHd, fTh, fTb, fTe;
  std::vector<Poly> ft;   // per-layer forward time, integer ns (the collector's t_l(x))
  // encoder-decoder: the same series on the 2-D key (x, xt)
  bool two_d = false;
  std::vector<Poly2> fa2, fy2, ft2;
  Poly2 fE2, fHd2, fTh2, fTb2, fTe2;
  void fit(const std::vector<Sample>& samples, int degree);
  void fit2(const std::vector<Sample>& samples, int degree);
  Series predict(int64_t x) const;
  Series predict2(int64_t x, int64_t xt) const;
  std::vector<int64_t> predict_cost2(int64_t x, int64_t xt) const;
  // Recompute cost per layer at x: the fitted forward time in ns, at least 1.
  std::vector<int64_t> predict_cost(int64_t x) const;
};

}  // namespace mimose
