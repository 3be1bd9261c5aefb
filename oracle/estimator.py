"""ORACLE (test infrastructure only): the lightning memory estimator.

PAPER.md §IV-C P:162 "the sizes of activation tensors ... are almost
polynomially correlated to the size of input tensors, and it is at most
quadratic"; "we finally choose the polynomial regression model";
§VI-E P:302-309 and Tables IV/V: quadratic (n=2) fitted on ~10 samples.

Reading R-A18: ordinary least squares with intercept, unweighted,
on t = x / x_ref (x_ref = largest sample x), degree 2 (fewer distinct x ->
degree = #distinct - 1); predictions are rounded half-to-even to integer
bytes plus a non-negative margin = the largest training under-prediction.

The least-squares step is the library routine numpy.linalg.lstsq.
Pinned by: exact recovery of integer polynomials (incl. extrapolation),
degree-1 / constant data, duplicate samples, fallback degrees
(tests/test_oracle_planning.py).
"""
from __future__ import annotations

from typing import Sequence

import numpy as np


class Quadratic:
    def __init__(self, xs: Sequence[int], ys: Sequence[int], degree: int = 2):
        xs = np.asarray(xs, np.float64)
        ys = np.asarray(ys, np.float64)
        if xs.size == 0:
            raise ValueError("no samples")
        n_distinct = len(set(xs.tolist()))
        self.degree = min(degree, n_distinct - 1)
        self.x_ref = float(xs.max())
        t = xs / self.x_ref
        A = np.stack([t ** k for k in range(self.degree + 1)], axis=1)
        self.coef = np.linalg.lstsq(A, ys, rcond=None)[0]
        fit = np.array([self._round(self._f(x)) for x in xs])
        self.margin = int(max(0, int((ys - fit).max())))

    def _f(self, x: float) -> float:
        t = float(x) / self.x_ref
        acc = 0.0
        for c in self.coef[::-1]:           # Horner
            acc = acc * t + float(c)
        return acc

    @staticmethod
    def _round(v: float) -> int:
        return int(np.rint(v))              # round half to even

    def predict(self, x: int) -> int:
        return self._round(self._f(x)) + self.margin


class Estimator:
    """One quadratic per collected series: d_l and a_l / y_l per layer, E, Hd,
    Th, Tb, Te (reading R-A20); C is measured exactly."""

    def __init__(self, samples, degree: int = 2):
        xs = [s["x"] for s in samples]
        self.C = samples[0]["C"]
        L = len(samples[0]["a"])
        self.L = L
        self.fa = [Quadratic(xs, [s["a"][l] for s in samples], degree) for l in range(L)]
        self.fy = [Quadratic(xs, [s["y"][l] for s in samples], degree) for l in range(L)]
        self.f = {k: Quadratic(xs, [s[k] for s in samples], degree)
                  for k in ("E", "Hd", "Th", "Tb", "Te")}

    def predict(self, x: int):
        a = [f.predict(x) for f in self.fa]
        y = [f.predict(x) for f in self.fy]
        out = {k: f.predict(x) for k, f in self.f.items()}
        out.update(C=self.C, a=a, y=y, d=[ai - yi for ai, yi in zip(a, y)])
        return out


# --------------------------------------------------------------------------
# 2-D key (reading A32): an encoder-decoder step has two
# input sizes, x = numel(source ids) and x_t = numel(target ids) (P:73's input
# size, one per input tensor).  Each series is fitted by an at most quadratic
# bivariate polynomial ("at most quadratic", P:164 polynomial regression)
# in s = x / x_ref, t = x_t / t_ref: features [1, s, t, s^2, s t, t^2]
# (degree 2, needs 6 distinct pairs of full rank), else [1, s, t] (degree 1,
# 3 non-collinear pairs), else the constant.  Least squares by the library
# routine numpy.linalg.lstsq; integer prediction rounded half-to-even plus the
# non-negative residual margin, as in 1-D.
# --------------------------------------------------------------------------

def _feats2(s, t, degree):
    cols = [np.ones_like(s)]
    if degree >= 1:
        cols += [s, t]
    if degree >= 2:
        cols += [s * s, s * t, t * t]
    return np.stack(cols, axis=1)


class Quadratic2D:
    def __init__(self, xs, ts, ys, degree: int = 2):
        xs, ts, ys = (np.asarray(v, np.float64) for v in (xs, ts, ys))
        self.x_ref, self.t_ref = float(xs.max()), float(ts.max())
        s, t = xs / self.x_ref, ts / self.t_ref
        pts = {(float(a), float(b)) for a, b in zip(xs, ts)}
        deg = degree
        while deg > 0:
            A = _feats2(s, t, deg)
            need = A.shape[1]
            if len(pts) >= need and np.linalg.matrix_rank(A) == need:
                break
            deg -= 1
        self.degree = deg
        A = _feats2(s, t, deg)
        self.coef = np.linalg.lstsq(A, ys, rcond=None)[0]
        fit = np.array([self._round(self._f(a, b)) for a, b in zip(xs, ts)])
        self.margin = int(max(0, int((ys - fit).max())))

    def _f(self, x, xt) -> float:
        s, t = float(x) / self.x_ref, float(xt) / self.t_ref
        f = [1.0, s, t, s * s, s * t, t * t][:len(self.coef)]
        return float(sum(float(c) * v for c, v in zip(self.coef, f)))

    @staticmethod
    def _round(v: float) -> int:
        return int(np.rint(v))

    def predict(self, x: int, xt: int) -> int:
        return self._round(self._f(x, xt)) + self.margin


class Estimator2D:
    """Estimator of an encoder-decoder's series on the 2-D key (x, x_t)."""

    def __init__(self, samples, degree: int = 2):
        xs = [s["x"] for s in samples]
        ts = [s["xt"] for s in samples]
        self.C = samples[0]["C"]
        L = len(samples[0]["a"])
        self.fa = [Quadratic2D(xs, ts, [s["a"][l] for s in samples], degree) for l in range(L)]
        self.fy = [Quadratic2D(xs, ts, [s["y"][l] for s in samples], degree) for l in range(L)]
        self.f = {k: Quadratic2D(xs, ts, [s[k] for s in samples], degree) for k in ("E", "Hd", "Th", "Tb", "Te")}

    def predict(self, x: int, xt: int):
        a = [f.predict(x, xt) for f in self.fa]
        y = [f.predict(x, xt) for f in self.fy]
        out = {k: f.predict(x, xt) for k, f in self.f.items()}
        out.update(C=self.C, a=a, y=y, d=[ai - yi for ai, yi in zip(a, y)])
        return out
