"""Pins of the NEXT-3 / NEXT-4 oracles (oracle/scaling.py; R26, R27)
against what the mathematics and library routines fix: an exactly
representable linear model is recovered with zero deviance; the residual is
orthogonal to the design (normal equations) and the deviance equals
R-style deviance from statsmodels-free closed forms; Spearman / Kendall equal
scipy's on tie-free and tied data; identical and reversed rankings give +1 / -1;
a hand-counted 4-element example."""
from __future__ import annotations

import math

import numpy as np
import pytest

from oracle import scaling as Sc


def test_glm_exact_polynomial_zero_deviance():
    N = np.arange(32, 2049, 32, dtype=np.float64)
    Z = np.stack([np.ones_like(N), N, N**2], axis=1)
    c_true = np.array([[3.0, -1.0], [0.5, 2.0], [0.25, 0.0]])
    Y = Z @ c_true
    coef, dev, null = Sc.glm_gaussian(Z, Y)
    assert np.allclose(coef, c_true, rtol=1e-9, atol=1e-9)
    assert np.all(dev <= 1e-12 * null)


def test_glm_normal_equations_and_deviances():
    rng = np.random.default_rng(3)
    n, k = 200, 4
    Z = np.concatenate([np.ones((n, 1)), rng.normal(size=(n, k - 1))], axis=1)
    Y = rng.normal(size=(n, 3)) + Z @ rng.normal(size=(k, 3))
    coef, dev, null = Sc.glm_gaussian(Z, Y)
    res = Y - Z @ coef
    assert np.allclose(Z.T @ res, 0.0, atol=1e-9)                   # normal equations
    assert np.allclose(dev, (res**2).sum(axis=0), rtol=1e-12)
    assert np.allclose(null, ((Y - Y.mean(axis=0)) ** 2).sum(axis=0), rtol=1e-12)
    # intercept-only model: deviance == null deviance
    c1, d1, n1 = Sc.glm_gaussian(np.ones((n, 1)), Y)
    assert np.allclose(d1, n1, rtol=1e-12)
    assert np.allclose(c1[0], Y.mean(axis=0), rtol=1e-12)


def test_glm_single_predictor_closed_form():
    # simple regression: slope = cov(x, y) / var(x), intercept = ybar - slope * xbar
    x = np.array([1.0, 2.0, 4.0, 7.0, 11.0])
    y = np.array([2.0, 3.0, 7.0, 8.0, 15.0])
    coef, dev, _ = Sc.glm_gaussian(np.stack([np.ones(5), x], axis=1), y)
    xb, yb = x.mean(), y.mean()
    slope = ((x - xb) * (y - yb)).sum() / ((x - xb) ** 2).sum()
    assert np.isclose(coef[1, 0], slope, rtol=1e-12)
    assert np.isclose(coef[0, 0], yb - slope * xb, rtol=1e-12)


def test_rank_similarity_hand_example():
    a = [0.1, 0.4, 0.4, 0.9]
    b = [1.0, 3.0, 2.0, 4.0]
    # pairs: (0,1) C, (0,2) C, (0,3) C, (1,2) Ta (a tie, b differs), (1,3) C, (2,3) C -> C=5, D=0, Ta=1, Tb=0
    assert math.isclose(Sc.kendall_tau_b(a, b), 5 / math.sqrt(6 * 5), rel_tol=1e-15)
    assert list(Sc.midranks(a)) == [1.0, 2.5, 2.5, 4.0]


def test_rank_similarity_special_cases():
    rng = np.random.default_rng(1)
    a = rng.normal(size=30)
    assert math.isclose(Sc.spearman(a, a), 1.0, rel_tol=1e-14)
    assert math.isclose(Sc.kendall_tau_b(a, -a), -1.0, rel_tol=1e-14)
    assert math.isclose(Sc.spearman(a, np.exp(a)), 1.0, rel_tol=1e-14)   # monotone transform
    assert math.isnan(Sc.spearman(np.ones(5), a[:5]))
    assert math.isnan(Sc.kendall_tau_b(np.ones(5), a[:5]))


@pytest.mark.parametrize("ties", [False, True])
def test_rank_similarity_vs_scipy(ties):
    stats = pytest.importorskip("scipy.stats")
    rng = np.random.default_rng(7 + ties)
    for p in (5, 20, 64):
        a = rng.normal(size=p)
        b = a + rng.normal(size=p)
        if ties:
            a, b = np.round(a * 2) / 2, np.round(b)
        assert math.isclose(Sc.spearman(a, b), stats.spearmanr(a, b)[0], rel_tol=1e-12, abs_tol=1e-15)
        assert math.isclose(Sc.kendall_tau_b(a, b), stats.kendalltau(a, b)[0], rel_tol=1e-12, abs_tol=1e-15)


def test_log_size_design_closed_form():
    """Sizes 2^5..2^11: log2 = 5..11 exactly, mean 8, sample sd sqrt(28/6); rows 1, u, u^2, u^3."""
    Z = Sc.log_size_design(2.0 ** np.arange(5, 12))
    u = (np.arange(5, 12) - 8.0) / math.sqrt(28.0 / 6.0)
    assert np.allclose(Z, np.stack([np.ones(7), u, u ** 2, u ** 3]), rtol=1e-15, atol=1e-15)


def test_prediction_error_closed_form():
    y = np.array([1.0, 2.0, 3.0, 4.0])
    mse, ex = Sc.prediction_error(y + np.array([0.5, -0.5, 0.5, -0.5]), y)
    assert mse == 0.25 and ex == pytest.approx(1.0 - 0.25 / 1.25, rel=1e-15)
    assert math.isnan(Sc.prediction_error(np.ones(3), np.full(3, 2.0))[1])
