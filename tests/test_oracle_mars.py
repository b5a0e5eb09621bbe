"""Pins of the MARS oracle (oracle/mars.py; R28) against what the
definition and exact arithmetic fix: recovery of an exact one-knot hinge
model (terms, coefficients, zero residual, the useless mirror hinge pruned);
lines fitted exactly with the lowest-knot tie rule; the forward step's
argmin checked by exact rational least squares on tiny integer data; GCV's
closed form; an additive two-predictor model recovered exactly."""
from __future__ import annotations

from fractions import Fraction

import numpy as np

from oracle import mars as Ms


def test_one_knot_hinge_recovered_and_mirror_pruned():
    x = np.arange(0.0, 21.0)
    y = 3.0 + 2.0 * np.maximum(0.0, x - 5.0)
    m = Ms.mars_fit(x[None, :], y)
    assert m["forward"] == [None, (0, 5.0, 1), (0, 5.0, -1)]
    assert m["terms"] == [None, (0, 5.0, 1)]                  # h(5 - x) has zero coefficient: pruned
    assert np.allclose(m["coef"], [3.0, 2.0], atol=1e-12)
    assert m["rss"] < 1e-20 and abs(m["rsq"] - 1.0) < 1e-15


def test_line_uses_lowest_knot_and_is_exact():
    x = np.array([0.0, 1.0, 3.0, 4.0, 8.0, 9.0])
    y = 1.5 - 0.25 * x
    m = Ms.mars_fit(x[None, :], y)
    assert m["forward"][1] == (0, 1.0, 1)                     # every knot fits exactly: the lowest wins
    assert np.allclose(Ms.mars_predict(m, x[None, :]), y, atol=1e-12)


def _rss_exact(cols, y):
    """Exact least-squares RSS with rational arithmetic (normal equations by Gauss-Jordan)."""
    k = len(cols)
    G = [[sum(Fraction(a) * Fraction(b) for a, b in zip(cols[i], cols[j])) for j in range(k)] for i in range(k)]
    rhs = [sum(Fraction(a) * Fraction(b) for a, b in zip(cols[i], y)) for i in range(k)]
    piv = []
    A = [row[:] + [r] for row, r in zip(G, rhs)]
    r0 = 0
    for c in range(k):
        p = next((i for i in range(r0, k) if A[i][c] != 0), None)
        if p is None:
            continue
        A[r0], A[p] = A[p], A[r0]
        A[r0] = [v / A[r0][c] for v in A[r0]]
        for i in range(k):
            if i != r0 and A[i][c] != 0:
                A[i] = [a - A[i][c] * b for a, b in zip(A[i], A[r0])]
        piv.append(c)
        r0 += 1
    coef = [Fraction(0)] * k
    for i, c in enumerate(piv):
        coef[c] = A[i][k]
    res = [Fraction(yy) - sum(coef[j] * Fraction(cols[j][i]) for j in range(k)) for i, yy in enumerate(y)]
    return sum(r * r for r in res)


def test_first_forward_step_is_the_exact_argmin():
    rng = np.random.default_rng(5)
    for trial in range(6):
        n = 10
        X = rng.integers(0, 6, (2, n)).astype(float)
        y = rng.integers(-5, 6, n).astype(float)
        m = Ms.mars_fit(X, y, thresh=0.0, nk=3)
        best = None
        for v in range(2):
            for t in Ms.candidate_knots(X[v]):
                cols = [[1.0] * n, list(np.maximum(0, X[v] - t)), list(np.maximum(0, t - X[v]))]
                r = _rss_exact(cols, list(y))
                if best is None or r < best[0]:
                    best = (r, v, float(t))
        if best is None or len(m["forward"]) < 3:
            continue
        assert m["forward"][1] == (best[1], best[2], 1), (trial, m["forward"], best)


def test_gcv_closed_form():
    x = np.linspace(0, 10, 40)
    rng = np.random.default_rng(2)
    y = np.maximum(0, x - 4) + 0.1 * rng.normal(size=40)
    m = Ms.mars_fit(x[None, :], y)
    M = len(m["terms"])
    C = M + 2.0 * (M - 1) / 2.0
    assert np.isclose(m["gcv"], (m["rss"] / 40) / (1 - C / 40) ** 2, rtol=1e-12)


def test_additive_two_predictors_recovered():
    g = np.arange(0.0, 10.0)
    x0, x1 = np.meshgrid(g, g)
    X = np.stack([x0.ravel(), x1.ravel()])
    y = np.maximum(0.0, X[0] - 3.0) + 2.0 * np.maximum(0.0, 7.0 - X[1])
    m = Ms.mars_fit(X, y)
    assert (0, 3.0, 1) in m["terms"] and (1, 7.0, -1) in m["terms"]
    assert np.allclose(Ms.mars_predict(m, X), y, atol=1e-10)
