"""Pins of the partial-dependence oracle (oracle/pdep.py) against what the
definition fixes (R23, R24): closed forms of
the grid, the exact step function of a one-split forest, constancy for a
predictor no split uses, and additivity over disjoint tree ranges."""
from __future__ import annotations

import numpy as np
import pytest

from oracle import oracle as O
from oracle import pdep as PD


def test_grid_closed_forms():
    assert PD.pd_grid(np.array([3.0, 1.0, 2.0, 2.0])).tolist() == [1.0, 2.0, 3.0]
    v = PD.pd_grid(np.arange(100, dtype=np.float64))  # 100 distinct -> 51 points, step 99/50
    assert len(v) == 51 and v[0] == 0.0 and v[-1] == 99.0
    assert np.allclose(np.diff(v), 99.0 / 50, rtol=1e-14)
    assert PD.pd_grid(np.full(7, 4.5)).tolist() == [4.5]                      # constant column: G = 1
    assert PD.pd_grid(np.array([-0.0, 0.0, 1.0])).tolist() == [0.0, 1.0]      # -0 == +0 (R18)
    assert len(PD.pd_grid(np.arange(10.0), n_pt=4)) == 4


def _stump_data(n=200, p=4, seed=3):
    rng = np.random.default_rng(seed)
    X = rng.normal(size=(p, n))
    y = np.where(X[1] > 0.2, 5.0, -1.0) + 0.01 * rng.normal(size=n)
    return X, y


def test_one_split_forest_is_an_exact_step():
    X, y = _stump_data()
    p, n = X.shape
    f = O.fit(X, y, ntree=1, mtry=p, nodesize=n - 1, seed=11)   # root splits once, children are leaves
    t = f.tree(0)
    assert t["feature"][0] == 1 and len(t["feature"]) == 3
    thr = t["thr"][0]
    vl, vr = t["value"][t["left"][0]], t["value"][t["left"][0] + 1]
    grid = np.array([X[1].min(), thr, np.nextafter(thr, np.inf), X[1].max()])
    _, pd = PD.partial_dependence(f, X, 1, grid)
    assert np.allclose(pd, [vl, vl, vr, vr], rtol=1e-13, atol=0)    # every row goes the same way
    # any other predictor: constant = mean prediction (n_L vl + n_R vr) / n over the rows of X
    nl = int((X[1] <= thr).sum())
    _, pd0 = PD.partial_dependence(f, X, 0, PD.pd_grid(X[0], 9))
    assert np.allclose(pd0, (nl * vl + (n - nl) * vr) / n, rtol=1e-13, atol=0)


def test_unused_predictor_is_flat_and_equals_mean_prediction():
    rng = np.random.default_rng(7)
    p, n = 5, 300
    X = rng.normal(size=(p, n))
    X[4] = 1.0                                   # constant: no split can use it
    y = X[0] * 2 + np.sin(X[2]) + 0.1 * rng.normal(size=n)
    f = O.fit(X, y, ntree=8, seed=5)
    used = set()
    for i in range(8):
        used |= set(int(v) for v in f.tree(i)["feature"] if v >= 0)
    assert 4 not in used
    grid = np.linspace(-3, 3, 11)
    s, pd = PD.partial_dependence(f, X, 4, grid)
    assert np.all(s == s[0])
    assert np.isclose(pd[0], f.predict_sum(X).mean() / 8, rtol=1e-13)
    # a used predictor is not flat on this data
    _, pd0 = PD.partial_dependence(f, X, 0, PD.pd_grid(X[0], 11))
    assert pd0.max() - pd0.min() > 1.0


def test_additive_over_disjoint_tree_ranges():
    rng = np.random.default_rng(9)
    p, n = 4, 150
    X = rng.normal(size=(p, n))
    y = X[1] - X[3] ** 2 + 0.1 * rng.normal(size=n)
    full = O.fit(X, y, ntree=6, seed=2)
    a = O.fit(X, y, ntree=6, seed=2, tree_begin=0, tree_end=2)
    b = O.fit(X, y, ntree=6, seed=2, tree_begin=2, tree_end=6)
    grid = PD.pd_grid(X[3], 7)
    sf, _ = PD.partial_dependence(full, X, 3, grid)
    sa, _ = PD.partial_dependence(a, X, 3, grid)
    sb, _ = PD.partial_dependence(b, X, 3, grid)
    assert np.allclose(sa + sb, sf, rtol=1e-13, atol=0)
