// See planning.h.  Compiled with -ffp-contract=off so the fp64 regression is
// evaluated operation by operation (no fused multiply-add reassociation).
#include "planning.h"

#include <algorithm>
#include <cmath>
#include <set>

namespace mimose {

void Poly::fit(const std::vector<int64_t>& xs, const std::vector<int64_t>& ys, int max_degree) {
  std::set<int64_t> distinct(xs.begin(), xs.end());
  degree = std::min<int>(max_degree, (int)distinct.size() - 1);
  if (degree < 0) degree = 0;
  x_ref = 1.0;
  for (int64_t x : xs) x_ref = std::max(x_ref, (double)x);
  const int n = degree + 1;
  double A[3][4] = {{0}};
  for (size_t i = 0; i < xs.size(); ++i) {
    const double t = (double)xs[i] / x_ref;
    double pw[3] = {1.0, t, t * t};
    for (int r = 0; r < n; ++r) {
      for (int c = 0; c < n; ++c) A[r][c] += pw[r] * pw[c];
      A[r][n] += pw[r] * (double)ys[i];
    }
  }
  for (int col = 0; col < n; ++col) {          // partial pivoting, fixed order
    int piv = col;
    for (int r = col + 1; r < n; ++r)
      if (std::fabs(A[r][col]) > std::fabs(A[piv][col])) piv = r;
    if (piv != col)
      for (int c = 0; c <= n; ++c) std::swap(A[col][c], A[piv][c]);
    for (int r = col + 1; r < n; ++r) {
      const double f = A[r][col] / A[col][col];
      for (int c = col; c <= n; ++c) A[r][c] -= f * A[col][c];
    }
  }
  for (int r = n - 1; r >= 0; --r) {
    double v = A[r][n];
    for (int c = r + 1; c < n; ++c) v -= A[r][c] * coef[c];
    coef[r] = v / A[r][r];
  }
  for (int r = n; r < 3; ++r) coef[r] = 0.0;
  margin = 0;
  for (size_t i = 0; i < xs.size(); ++i) {
    const int64_t fitv = (int64_t)std::nearbyint(eval(xs[i]));
    margin = std::max<int64_t>(margin, ys[i] - fitv);
  }
}

double Poly::eval(int64_t x) const {
  const double t = (double)x / x_ref;
  double acc = 0.0;
  for (int k = degree; k >= 0; --k) acc = acc * t + coef[k];   // Horner
  return acc;
}

int64_t Poly::predict(int64_t x) const { return (int64_t)std::nearbyint(eval(x)) + margin; }

static int solve_normal(double (*A)[7], int n, double* coef) {
  // Gaussian elimination with partial pivoting in a fixed order; returns 0 if a
  // pivot vanishes relative to the diagonal scale (rank deficient)
  double scale = 0.0;
  for (int r = 0; r < n; ++r) scale = std::max(scale, std::fabs(A[r][r]));
  for (int col = 0; col < n; ++col) {
    int piv = col;
    for (int r = col + 1; r < n; ++r)
      if (std::fabs(A[r][col]) > std::fabs(A[piv][col])) piv = r;
    if (!(std::fabs(A[piv][col]) > 1e-10 * scale)) return 0;
    if (piv != col)
      for (int c = 0; c <= n; ++c) std::swap(A[col][c], A[piv][c]);
    for (int r = col + 1; r < n; ++r) {
      const double f = A[r][col] / A[col][col];
      for (int c = col; c <= n; ++c) A[r][c] -= f * A[col][c];
    }
  }
  for (int r = n - 1; r >= 0; --r) {
    double v = A[r][n];
    for (int c = r + 1; c < n; ++c) v -= A[r][c] * coef[c];
    coef[r] = v / A[r][r];
  }
  return 1;
}

void Poly2::fit(const std::vector<int64_t>& xs, const std::vector<int64_t>& ts, const std::vector<int64_t>& ys,
                int max_degree) {
  std::set<std::pair<int64_t, int64_t>> distinct;
  for (size_t i = 0; i < xs.size(); ++i) distinct.insert({xs[i], ts[i]});
  x_ref = t_ref = 1.0;
  for (size_t i = 0; i < xs.size(); ++i) {
    x_ref = std::max(x_ref, (double)xs[i]);
    t_ref = std::max(t_ref, (double)ts[i]);
  }
  for (degree = std::min(max_degree, 2); degree >= 0; --degree) {
    nf = degree == 2 ? 6 : degree == 1 ? 3 : 1;
    if ((int)distinct.size() < nf) continue;
    double A[6][7] = {{0}};
    for (size_t i = 0; i < xs.size(); ++i) {
      const double s = (double)xs[i] / x_ref, t = (double)ts[i] / t_ref;
      const double f[6] = {1.0, s, t, s * s, s * t, t * t};
      for (int r = 0; r < nf; ++r) {
        for (int c = 0; c < nf; ++c) A[r][c] += f[r] * f[c];
        A[r][nf] += f[r] * (double)ys[i];
      }
    }
    for (int r = 0; r < 6; ++r) coef[r] = 0.0;
    if (solve_normal(A, nf, coef)) break;
  }
  if (degree < 0) {                          // no pairs at all: constant 0
    degree = 0;
    nf = 1;
    coef[0] = 0.0;
  }
  margin = 0;
  for (size_t i = 0; i < xs.size(); ++i)
    margin = std::max<int64_t>(margin, ys[i] - (int64_t)std::nearbyint(eval(xs[i], ts[i])));
}

double Poly2::eval(int64_t x, int64_t xt) const {
  const double s = (double)x / x_ref, t = (double)xt / t_ref;
  const double f[6] = {1.0, s, t, s * s, s * t, t * t};
  double acc = 0.0;
  for (int k = 0; k < nf; ++k) acc += coef[k] * f[k];
  return acc;
}

int64_t Poly2::predict(int64_t x, int64_t xt) const { return (int64_t)std::nearbyint(eval(x, xt)) + margin; }

int64_t predicted_peak(const Series& s, uint64_t mask) {
  const int L = (int)s.a.size();
  const int64_t base = s.C + s.E;
  int64_t pk = base + s.Te;
  int64_t S = 0;
  std::vector<int64_t> prefix(L);
  for (int l = 0; l < L; ++l) {
    prefix[l] = S;
    pk = std::max(pk, base + S + s.a[l]);                 // forward of layer l
    S += ((mask >> l) & 1) ? s.y[l] : s.a[l];
  }
  pk = std::max(pk, base + S + s.Hd + s.Th);             // head backward
  for (int l = 0; l < L; ++l)                            // layer backward (recompute if dropped)
    pk = std::max(pk, base + prefix[l] + (s.a[l] - s.y[l]) + s.Tb);
  return pk;
}

PlanResult plan_greedy(const Series& s, int64_t budget, int64_t reserve, int bnum, int bden) {
  const int L = (int)s.a.size();
  const int64_t limit = budget - reserve;
  std::vector<int64_t> est(L);
  for (int l = 0; l < L; ++l) est[l] = s.a[l] - s.y[l];            // A4: droppable bytes
  // lines 2-12: buckets over candidates 0..L-2 (A12)
  std::vector<int> order;
  for (int l = 0; l + 1 < L; ++l) order.push_back(l);
  std::stable_sort(order.begin(), order.end(), [&](int a, int b) { return est[a] > est[b]; });  // A5
  std::vector<std::vector<int>> buckets;
  for (size_t i = 0; i < order.size();) {
    const int head = order[i++];
    std::vector<int> b{head};
    while (i < order.size() && (int64_t)bden * est[order[i]] > (int64_t)bnum * est[head]) b.push_back(order[i++]);  // A6
    std::sort(b.begin(), b.end());                                 // A7
    buckets.push_back(b);
  }
  auto bmax = [&](const std::vector<int>& b) {
    int64_t m = INT64_MIN;
    for (int l : b) m = std::max(m, est[l]);
    return m;
  };
  uint64_t mask = 0;
  int64_t pk = predicted_peak(s, 0);
  int64_t excess = pk - limit;                                     // line 13 (A1)
  for (;;) {
    bool exhausted = false;
    while (excess > 0) {                                           // line 14 (A10)
      if (buckets.empty()) { exhausted = true; break; }
      int pick = -1;                                               // bucket index
      int64_t best = INT64_MAX;
      for (size_t bi = 0; bi < buckets.size(); ++bi) {             // line 15
        const int64_t m = bmax(buckets[bi]);
        if (m > excess && m < best) { best = m; pick = (int)bi; }  // line 19 (A8: nearest)
      }
      if (pick < 0) pick = 0;                                      // line 17 (A9)
      const int l = buckets[pick].front();
      mask |= 1ull << l;                                           // line 20
      buckets[pick].erase(buckets[pick].begin());
      if (buckets[pick].empty()) buckets.erase(buckets.begin() + pick);
      excess -= est[l];                                            // line 21 (A2)
    }
    if (exhausted) break;
    pk = predicted_peak(s, mask);                                  // A13 verify
    excess = pk - limit;
    if (excess <= 0) return {true, mask, pk};
  }
  if (L > 0 && !((mask >> (L - 1)) & 1)) {                         // A12 last resort
    mask |= 1ull << (L - 1);
    pk = predicted_peak(s, mask);
    if (pk <= limit) return {true, mask, pk};
  }
  return {false, mask, predicted_peak(s, mask)};
}

namespace {
// Least total recompute cost of layers [l0, L) given `S0` stack bytes below l0,
// such that every remaining event fits R (relative to C + E): layer l's
// forward / backward events S_l + max(a_l, a_l - y_l + Tb) and the head event
// S_L + Hd + Th.  Forward DP over layers with the 2-D Pareto front of
// (stack bytes, cost): a state with no more bytes and no more cost than
// another makes every completion at least as cheap and as feasible.
int64_t min_cost_from(const Series& s, const std::vector<int64_t>& cost, const std::vector<int64_t>& suf_y,
                      int l0, int64_t S0, int64_t R) {
  const int L = (int)s.a.size();
  std::vector<std::pair<int64_t, int64_t>> cur{{S0, 0}}, nxt;
  for (int l = l0; l < L && !cur.empty(); ++l) {
    const int64_t need = std::max(s.a[l], s.a[l] - s.y[l] + s.Tb);
    nxt.clear();
    for (auto& [S, c] : cur) {
      if (S + need > R) continue;
      if (S + s.y[l] + suf_y[l + 1] + s.Hd + s.Th <= R) nxt.push_back({S + s.y[l], c + cost[l]});
      if (S + s.a[l] + suf_y[l + 1] + s.Hd + s.Th <= R) nxt.push_back({S + s.a[l], c});
    }
    std::sort(nxt.begin(), nxt.end());
    cur.clear();
    int64_t best = INT64_MAX;
    for (auto& st : nxt)
      if (st.second < best) { cur.push_back(st); best = st.second; }
  }
  int64_t best = INT64_MAX;
  for (auto& [S, c] : cur)
    if (S + s.Hd + s.Th <= R) best = std::min(best, c);
  return best;
}
}  // namespace

PlanResult plan_exact_cost(const Series& s, const std::vector<int64_t>& cost_in, int64_t budget, int64_t reserve) {
  const int L = (int)s.a.size();
  const int64_t base = s.C + s.E;
  const int64_t R = budget - reserve - base;
  const uint64_t all = L >= 64 ? ~0ull : ((1ull << L) - 1);
  std::vector<int64_t> cost(L), suf_y(L + 1, 0);
  for (int l = 0; l < L; ++l) cost[l] = std::max<int64_t>(1, cost_in[l]);
  for (int l = L - 1; l >= 0; --l) suf_y[l] = suf_y[l + 1] + s.y[l];
  auto mc = [&](int l0, int64_t S0, int64_t lim) {
    return s.Te <= lim ? min_cost_from(s, cost, suf_y, l0, S0, lim) : INT64_MAX;
  };
  // 1. the least total cost
  const int64_t cstar = mc(0, 0, R);
  if (cstar == INT64_MAX) return {false, all, predicted_peak(s, all)};
  // 2. the lowest peak among least-cost sets: the smallest limit P <= R under
  //    which the least cost is still cstar (it only rises as P falls)
  int64_t lo = 0, hi = R;
  while (lo < hi) {
    const int64_t mid = lo + (hi - lo) / 2;
    if (mc(0, 0, mid) == cstar) hi = mid; else lo = mid + 1;
  }
  const int64_t P = hi;
  // 3. the lexicographically smallest sorted layer list among them: drop each
  //    layer in order whenever a completion with total cost cstar under P exists
  //    (all costs >= 1, so no least-cost list is a proper prefix of another)
  uint64_t mask = 0;
  int64_t S = 0, c = 0;
  for (int l = 0; l < L; ++l) {
    const int64_t rest = mc(l + 1, S + s.y[l], P);
    if (rest != INT64_MAX && c + cost[l] + rest == cstar) {
      mask |= 1ull << l;
      S += s.y[l];
      c += cost[l];
    } else {
      S += s.a[l];
    }
  }
  return {true, mask, base + P};
}

// Unit recompute cost: the same least-cost search with every cost 1 (fewest
// recomputed layers, then lowest peak, then lexicographic; reading A29).
PlanResult plan_exact(const Series& s, int64_t budget, int64_t reserve) {
  return plan_exact_cost(s, std::vector<int64_t>(s.a.size(), 1), budget, reserve);
}

void Estimator::fit(const std::vector<Sample>& smp, int degree) {
  const int L = (int)smp.front().a.size();
  std::vector<int64_t> xs;
  for (auto& s : smp) xs.push_back(s.x);
  auto series = [&](auto get) {
    std::vector<int64_t> v;
    for (auto& s : smp) v.push_back(get(s));
    return v;
  };
  C = smp.front().C;
  fa.assign(L, Poly());
  fy.assign(L, Poly());
  for (int l = 0; l < L; ++l) {
    fa[l].fit(xs, series([&](const Sample& s) { return s.a[l]; }), degree);
    fy[l].fit(xs, series([&](const Sample& s) { return s.y[l]; }), degree);
  }
  fE.fit(xs, series([](const Sample& s) { return s.E; }), degree);
  fHd.fit(xs, series([](const Sample& s) { return s.Hd; }), degree);
  fTh.fit(xs, series([](const Sample& s) { return s.Th; }), degree);
  fTb.fit(xs, series([](const Sample& s) { return s.Tb; }), degree);
  fTe.fit(xs, series([](const Sample& s) { return s.Te; }), degree);
  ft.assign(L, Poly());
  for (int l = 0; l < L; ++l)
    ft[l].fit(xs, series([&](const Sample& s) { return (int64_t)std::llround((double)s.t_ms[l] * 1e6); }), degree);
  fitted = true;
}

void Estimator::fit2(const std::vector<Sample>& smp, int degree) {
  const int L = (int)smp.front().a.size();
  std::vector<int64_t> xs, ts;
  for (auto& s : smp) { xs.push_back(s.x); ts.push_back(s.xt); }
  auto series = [&](auto get) {
    std::vector<int64_t> v;
    for (auto& s : smp) v.push_back(get(s));
    return v;
  };
  C = smp.front().C;
  fa2.assign(L, Poly2());
  fy2.assign(L, Poly2());
  ft2.assign(L, Poly2());
  for (int l = 0; l < L; ++l) {
    fa2[l].fit(xs, ts, series([&](const Sample& s) { return s.a[l]; }), degree);
    fy2[l].fit(xs, ts, series([&](const Sample& s) { return s.y[l]; }), degree);
    ft2[l].fit(xs, ts, series([&](const Sample& s) { return (int64_t)std::llround((double)s.t_ms[l] * 1e6); }),
               degree);
  }
  fE2.fit(xs, ts, series([](const Sample& s) { return s.E; }), degree);
  fHd2.fit(xs, ts, series([](const Sample& s) { return s.Hd; }), degree);
  fTh2.fit(xs, ts, series([](const Sample& s) { return s.Th; }), degree);
  fTb2.fit(xs, ts, series([](const Sample& s) { return s.Tb; }), degree);
  fTe2.fit(xs, ts, series([](const Sample& s) { return s.Te; }), degree);
  two_d = true;
  fitted = true;
}

Series Estimator::predict2(int64_t x, int64_t xt) const {
  Series s;
  s.C = C;
  s.E = fE2.predict(x, xt);
  s.Hd = fHd2.predict(x, xt);
  s.Th = fTh2.predict(x, xt);
  s.Tb = fTb2.predict(x, xt);
  s.Te = fTe2.predict(x, xt);
  for (size_t l = 0; l < fa2.size(); ++l) {
    s.a.push_back(fa2[l].predict(x, xt));
    s.y.push_back(fy2[l].predict(x, xt));
  }
  return s;
}

std::vector<int64_t> Estimator::predict_cost2(int64_t x, int64_t xt) const {
  std::vector<int64_t> c(ft2.size());
  for (size_t l = 0; l < ft2.size(); ++l) c[l] = std::max<int64_t>(1, (int64_t)std::nearbyint(ft2[l].eval(x, xt)));
  return c;
}

std::vector<int64_t> Estimator::predict_cost(int64_t x) const {
  std::vector<int64_t> c(ft.size());
  for (size_t l = 0; l < ft.size(); ++l) c[l] = std::max<int64_t>(1, (int64_t)std::nearbyint(ft[l].eval(x)));
  return c;
}

Series Estimator::predict(int64_t x) const {
  Series s;
  s.C = C;
  s.E = fE.predict(x);
  s.Hd = fHd.predict(x);
  s.Th = fTh.predict(x);
  s.Tb = fTb.predict(x);
  s.Te = fTe.predict(x);
  for (size_t l = 0; l < fa.size(); ++l) {
    s.a.push_back(fa[l].predict(x));
    s.y.push_back(fy[l].predict(x));
  }
  return s;
}

}  // namespace mimose
