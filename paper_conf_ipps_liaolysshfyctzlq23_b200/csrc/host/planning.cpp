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
struct ExactSearch {
  const Series& s;
  int L;
  int64_t R;           // limit - (C + E): room for stack + transients
  int k;               // drops to place
  std::vector<int64_t> need;   // per-layer transient on top of its prefix
  std::vector<int64_t> suf_a, suf_dmax;   // sum a_j and max (a_j - y_j) over j >= l
  bool found = false;
  int64_t best_pk = 0;
  uint64_t best_mask = 0;
  // Layers [l, L) remain; `left` drops still to place; prefix = stack bytes
  // below layer l; runmax = max over the constraints of layers < l.
  void dfs(int l, int left, int64_t prefix, int64_t runmax, uint64_t mask) {
    if (found && runmax >= best_pk) return;             // cannot beat the best peak
    if (l == L) {
      if (left) return;
      const int64_t pk = std::max(runmax, prefix + s.Hd + s.Th);
      if (pk > R) return;
      if (!found || pk < best_pk) { found = true; best_pk = pk; best_mask = mask; }
      return;
    }
    if (L - l < left) return;
    // even the `left` largest savings below cannot bring the head event under R
    if (prefix + suf_a[l] - (int64_t)left * suf_dmax[l] + s.Hd + s.Th > R) return;
    const int64_t here = prefix + need[l];              // layer l's forward / backward events
    if (here > R) return;                               // fixed by the choices below l
    const int64_t rm = std::max(runmax, here);
    if (left > 0) dfs(l + 1, left - 1, prefix + s.y[l], rm, mask | (1ull << l));   // drop first: lex order
    dfs(l + 1, left, prefix + s.a[l], rm, mask);
  }
};
}  // namespace

PlanResult plan_exact(const Series& s, int64_t budget, int64_t reserve) {
  const int L = (int)s.a.size();
  const int64_t base = s.C + s.E;
  ExactSearch x{s, L, budget - reserve - base, 0, {}};
  x.need.resize(L);
  for (int l = 0; l < L; ++l) x.need[l] = std::max(s.a[l], s.a[l] - s.y[l] + s.Tb);
  x.suf_a.assign(L + 1, 0);
  x.suf_dmax.assign(L + 1, 0);
  for (int l = L - 1; l >= 0; --l) {
    x.suf_a[l] = x.suf_a[l + 1] + s.a[l];
    x.suf_dmax[l] = std::max(x.suf_dmax[l + 1], s.a[l] - s.y[l]);
  }
  if (s.Te <= x.R) {
    for (int k = 0; k <= L && !x.found; ++k) {
      x.k = k;
      x.dfs(0, k, 0, s.Te, 0);
    }
  }
  if (!x.found) {
    const uint64_t all = L >= 64 ? ~0ull : ((1ull << L) - 1);
    return {false, all, predicted_peak(s, all)};
  }
  return {true, x.best_mask, base + x.best_pk};
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
  fitted = true;
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
