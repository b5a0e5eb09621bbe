"""Pins of the varimax oracle (oracle/varimax.py; R25) against
what the mathematics fixes: Kaiser's closed-form angle for two factors, an
orthogonal rotation that never lowers the varimax criterion, invariance of
the optimum under a prior orthogonal rotation, and simple structure as a
fixed point."""
from __future__ import annotations

import numpy as np

from oracle import varimax as V


def _kaiser_angle(x):
    """Two-factor optimum of the raw varimax criterion (Kaiser 1958):
    tan(4 phi) = (D - 2AB/p) / (C - (A^2 - B^2)/p)."""
    p = x.shape[0]
    u = x[:, 0] ** 2 - x[:, 1] ** 2
    v = 2 * x[:, 0] * x[:, 1]
    A, B = u.sum(), v.sum()
    C, D = (u * u - v * v).sum(), 2 * (u * v).sum()
    return np.arctan2(D - 2 * A * B / p, C - (A * A - B * B) / p) / 4


def _rot(phi):
    c, s = np.cos(phi), np.sin(phi)
    return np.array([[c, -s], [s, c]])


def test_two_factor_matches_kaiser_closed_form():
    rng = np.random.default_rng(4)
    x = rng.normal(size=(12, 2))
    z, T, it = V.varimax(x, normalize=False, eps=1e-15)
    phi = _kaiser_angle(x)
    zk = x @ _rot(phi)
    assert np.isclose(V.criterion(z), V.criterion(zk), rtol=1e-12)
    # same loadings up to column order and sign (the optimum is unique up to those)
    for perm in ([0, 1], [1, 0]):
        zz = zk[:, perm]
        sg = np.sign((zz * z).sum(axis=0))
        if np.allclose(zz * sg, z, atol=1e-7):
            break
    else:
        raise AssertionError("varimax optimum differs from Kaiser's angle")


def test_orthogonal_and_monotone():
    rng = np.random.default_rng(8)
    for p, k in [(30, 3), (60, 5), (16, 8)]:
        x = rng.normal(size=(p, k))
        z, T, it = V.varimax(x)
        assert np.allclose(T.T @ T, np.eye(k), atol=1e-12)
        assert np.allclose(z, x @ T, atol=1e-12)           # normalisation undone exactly (rows scaled back)
        xn = x / np.sqrt((x * x).sum(axis=1))[:, None]
        assert V.criterion(xn @ T) >= V.criterion(xn) - 1e-12
        assert 1 <= it <= 1000


def test_invariant_under_prior_rotation():
    rng = np.random.default_rng(12)
    x = rng.normal(size=(40, 4))
    Q, _ = np.linalg.qr(rng.normal(size=(4, 4)))
    z1, _, _ = V.varimax(x, eps=1e-14)
    z2, _, _ = V.varimax(x @ Q, eps=1e-14)
    # columns of z2 are a signed permutation of z1's
    M = np.abs(z1.T @ z2) / np.outer(np.linalg.norm(z1, axis=0), np.linalg.norm(z2, axis=0))
    assert np.allclose(np.sort(M.max(axis=1)), 1.0, atol=1e-6)


def test_simple_structure_is_a_fixed_point():
    x = np.zeros((9, 3))
    for i in range(9):
        x[i, i % 3] = 0.5 + 0.1 * i
    z, T, it = V.varimax(x)
    assert np.allclose(np.abs(T), np.eye(3), atol=1e-12)
    assert np.allclose(np.abs(z), np.abs(x), atol=1e-12)


def test_single_factor_is_returned_unchanged():
    x = np.arange(6.0).reshape(6, 1)
    z, T, it = V.varimax(x)
    assert np.array_equal(z, x) and T.shape == (1, 1) and it == 0
