"""CPU ORACLE -- MARS counter models (second half).

TEST INFRASTRUCTURE ONLY (see oracle/oracle.py header).

PAPER.md:138-145 (sec 4.1.3, eq. 4): f(x) = sum_i c_i B_i(x), B_i = the
intercept or a hinge max(0, x - c) / max(0, c - x) (the garbled "max(x-c)"
read as max(0, x - c), reading R19); P:173 ("we use MARS regressions to take
into account nonlinearities"), P:256 (R earth, "average R-squared of 0.99").
Reading R28 fixes the algorithm as Friedman's MARS with earth's defaults for
additive models (degree 1), restated step by step:

  forward pass
    basis = [1]; nk = min(200, max(20, 2 d)) + 1; thresh = 0.001
    candidates: every predictor v and every knot t in the distinct values of
      x_v other than its minimum and maximum; pair = (max(0, x_v - t), max(0, t - x_v))
    repeat while len(basis) + 2 <= nk:
      for each candidate: RSS of the least-squares fit of y on basis + pair   (library lstsq)
      best = the lowest (v, t) among the candidates whose RSS <= min RSS + tol * TSS
             (tol = 1e-12: mathematically tied candidates differ only by rounding)
      RSq(basis) = 1 - RSS / TSS  (TSS = sum (y - mean y)^2)
      if RSq(basis + best) - RSq(basis) < thresh: stop
      basis += best pair
      if RSq >= 1 - thresh: stop
  backward pass (penalty = 2, degree 1)
    GCV(S) = (RSS(S) / n) / (1 - C(S) / n)^2,  C(S) = |S| + penalty (|S| - 1) / 2
    S = all terms; best = S
    while |S| > 1: drop the non-intercept term whose removal gives the smallest RSS
                   (within tol * TSS -> the earliest term); if GCV(S) <= GCV(best) + tol * TSS / n: best = S
    (GCV ties within tol go to the smaller model)
  result: terms of best (v, t, dir), least-squares coefficients, RSS, GCV, RSq
"""
from __future__ import annotations

import numpy as np

TOL = 1e-12


def _rss(B: np.ndarray, y: np.ndarray) -> float:
    c = np.linalg.lstsq(B, y, rcond=None)[0]
    r = y - B @ c
    return float(r @ r)


def hinge(x: np.ndarray, t: float, direction: int) -> np.ndarray:
    return np.maximum(0.0, x - t) if direction > 0 else np.maximum(0.0, t - x)


def candidate_knots(x: np.ndarray) -> np.ndarray:
    u = np.unique(np.asarray(x, dtype=np.float64) + 0.0)
    return u[1:-1]


def mars_fit(X: np.ndarray, y: np.ndarray, nk: int | None = None, thresh: float = 0.001, penalty: float = 2.0):
    """X: (d, n) predictors, y: (n,).  Returns dict(terms=[(v, t, dir)], coef, rss, gcv, rsq, forward=[...])."""
    X = np.asarray(X, dtype=np.float64)
    y = np.asarray(y, dtype=np.float64)
    d, n = X.shape
    if nk is None:
        nk = min(200, max(20, 2 * d)) + 1
    tss = float(((y - y.mean()) ** 2).sum())
    terms = [None]                       # None = intercept
    cols = [np.ones(n)]
    rss = _rss(np.stack(cols, 1), y)
    knots = [candidate_knots(X[v]) for v in range(d)]
    while len(terms) + 2 <= nk and tss > 0:
        B = np.stack(cols, 1)
        cand = []
        for v in range(d):
            for t in knots[v]:
                r = _rss(np.concatenate([B, hinge(X[v], t, 1)[:, None], hinge(X[v], t, -1)[:, None]], 1), y)
                cand.append((r, v, float(t)))
        if not cand:
            break
        rmin = min(c[0] for c in cand)
        best = next(c for c in cand if c[0] <= rmin + TOL * tss)   # candidates are in (v, t) order
        if (1.0 - best[0] / tss) - (1.0 - rss / tss) < thresh:
            break
        _, v, t = best
        terms += [(v, t, 1), (v, t, -1)]
        cols += [hinge(X[v], t, 1), hinge(X[v], t, -1)]
        rss = best[0]
        if 1.0 - rss / tss >= 1.0 - thresh:
            break
    forward = list(terms)

    def gcv(r, m):
        C = m + penalty * (m - 1) / 2.0
        return (r / n) / (1.0 - C / n) ** 2

    S = list(range(len(terms)))
    best_S, best_g = list(S), gcv(rss, len(S))
    cur_rss = rss
    while len(S) > 1:
        cand = []
        for i in S[1:]:
            T = [j for j in S if j != i]
            cand.append((_rss(np.stack([cols[j] for j in T], 1), y), i))
        rmin = min(c[0] for c in cand)
        cur_rss, drop = next(c for c in cand if c[0] <= rmin + TOL * tss)
        S = [j for j in S if j != drop]
        g = gcv(cur_rss, len(S))
        if g <= best_g + TOL * tss / n:
            best_S, best_g = list(S), g
    Bb = np.stack([cols[j] for j in best_S], 1)
    coef = np.linalg.lstsq(Bb, y, rcond=None)[0]
    r = y - Bb @ coef
    rb = float(r @ r)
    return {"terms": [terms[j] for j in best_S], "coef": coef, "rss": rb, "gcv": best_g,
            "rsq": 1.0 - rb / tss if tss > 0 else 1.0, "forward": forward}


def mars_predict(model: dict, X: np.ndarray) -> np.ndarray:
    X = np.asarray(X, dtype=np.float64)
    out = np.zeros(X.shape[1])
    for c, term in zip(model["coef"], model["terms"]):
        out += c * (1.0 if term is None else hinge(X[term[0]], term[1], term[2]))
    return out
