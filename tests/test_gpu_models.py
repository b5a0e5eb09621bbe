"""GPU parity of the NEXT-3 / NEXT-4 kernels (models.cu) against the oracle
(oracle/scaling.py): gaussian GLM counter models (coefficients, fitted values,
residual and null deviance), the models on new rows, and the importance
ranking similarity (Spearman, Kendall tau-b; exact integer pair counts)."""
from __future__ import annotations

import math

import numpy as np
import pytest

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():
    pytest.skip("no CUDA device", allow_module_level=True)

import paper_conf_ipps_madougouvln16_b200 as bf  # noqa: E402
from oracle import scaling as Sc  # noqa: E402

DEV = torch.device("cuda:0")


def dev(a):
    return torch.from_numpy(np.ascontiguousarray(a)).to(DEV)


def _design(size, kind):
    s = (np.log2(size) - np.log2(size).mean()) / np.log2(size).std()
    cols = {"lin": [np.ones_like(s), s], "cubic": [np.ones_like(s), s, s**2, s**3],
            "mixed": [np.ones_like(s), s, s**2, np.sqrt(size / size.max()), size / size.max()]}[kind]
    return np.stack(cols, axis=0)  # (k, n)


# n: ragged, one CTA, many CTAs (grid-stride); r responses
@pytest.mark.parametrize("n,kind,r", [(24, "lin", 6), (129, "cubic", 8), (4096, "mixed", 40), (300001, "cubic", 3)])
def test_glm_parity(n, kind, r):
    rng = np.random.default_rng(n)
    size = 32.0 * rng.integers(1, 65, n)
    Z = _design(size, kind)
    k = Z.shape[0]
    Y = (rng.normal(size=(r, k)) @ Z) * 10.0 ** rng.uniform(0, 6, (r, 1)) + rng.normal(size=(r, n)) * 10.0 ** rng.uniform(-3, 3, (r, 1))
    g = bf.glm_gaussian(dev(Z), dev(Y))
    co, do, no = Sc.glm_gaussian(Z.T, Y.T)
    gc = g["coef"].cpu().numpy()
    fit_g, fit_o = gc @ Z, co.T @ Z
    scale = np.abs(Y).max(axis=1, keepdims=True)
    assert np.all(np.abs(fit_g - fit_o) <= 1e-10 * scale)
    assert np.allclose(g["null_deviance"].cpu().numpy(), no, rtol=1e-10)
    dg = g["deviance"].cpu().numpy()
    assert np.all(np.abs(dg - do) <= 1e-8 * do + 1e-12 * no)
    # the models on new rows
    Zn = _design(32.0 * rng.integers(1, 129, 777), kind)
    pn = bf.glm_predict(dev(Zn), g["coef"]).cpu().numpy()
    assert np.allclose(pn, gc @ Zn, rtol=1e-12, atol=1e-12 * np.abs(pn).max())


def test_glm_exact_polynomial_and_host_pointers():
    N = np.arange(32, 2049, 32, dtype=np.float64)
    Z = _design(N, "cubic")
    c_true = np.array([[3.0, -1.0, 0.5, 0.25], [1.0, 2.0, 0.0, -0.5]])
    Y = c_true @ Z
    g = bf.glm_gaussian(Z, Y)  # host numpy: staged by the library
    assert np.allclose(g["coef"], c_true, rtol=1e-10, atol=1e-10)
    assert np.all(g["deviance"] <= 1e-20 * g["null_deviance"] + 1e-20)


def test_glm_rank_deficient_rejected():
    N = np.arange(1, 101, dtype=np.float64)
    Z = np.stack([np.ones_like(N), N, 2 * N], axis=0)
    with pytest.raises(bf.BFError) as ei:
        bf.glm_gaussian(dev(Z), dev(N[None, :]))
    assert ei.value.code == -1


@pytest.mark.parametrize("p,ties", [(1, False), (2, False), (20, False), (64, True), (257, True), (3000, False)])
def test_rank_similarity_parity(p, ties):
    rng = np.random.default_rng(p + ties)
    a = rng.normal(size=p)
    b = a + rng.normal(size=p)
    if ties:
        a, b = np.round(a * 2) / 2, np.round(b)
    rho, tau = bf.rank_similarity(dev(a), dev(b))
    if p < 2:
        assert math.isnan(rho) and math.isnan(tau)
        return
    ro = Sc.spearman(a, b) if p <= 300 else None
    to = Sc.kendall_tau_b(a, b) if p <= 300 else None
    if ro is None:  # the plain oracle is O(p^2) Python: use its numpy restatement of the same formulas
        ra = np.array([(a < v).sum() + ((a == v).sum() + 1) / 2 for v in a])
        rb = np.array([(b < v).sum() + ((b == v).sum() + 1) / 2 for v in b])
        ro = float(np.corrcoef(ra, rb)[0, 1])
        sa, sb = np.sign(a[:, None] - a[None, :]), np.sign(b[:, None] - b[None, :])
        iu = np.triu_indices(p, 1)
        prod = (sa * sb)[iu]
        C, D = (prod > 0).sum(), (prod < 0).sum()
        Ta = ((sa[iu] == 0) & (sb[iu] != 0)).sum()
        Tb = ((sb[iu] == 0) & (sa[iu] != 0)).sum()
        to = (C - D) / math.sqrt((C + D + Ta) * (C + D + Tb))
    assert math.isclose(rho, ro, rel_tol=1e-12, abs_tol=1e-14)
    assert math.isclose(tau, to, rel_tol=1e-13, abs_tol=1e-15)
    # identical and reversed rankings
    r1, t1 = bf.rank_similarity(dev(a), dev(a))
    assert math.isclose(r1, 1.0, rel_tol=1e-14) and math.isclose(t1, 1.0, rel_tol=1e-14)


# ------------------------------------------------------------------ MARS (R28)
from oracle import mars as Ms  # noqa: E402


def _mars_cases():
    rng = np.random.default_rng(11)
    x = np.arange(0.0, 21.0)
    yield "hinge", x[None, :], 3.0 + 2.0 * np.maximum(0.0, x - 5.0)
    xs = rng.uniform(0, 10, 500)
    yield "noisy_1d", xs[None, :], np.sin(xs) + 0.3 * xs + 0.05 * rng.normal(size=500)
    X2 = rng.uniform(0, 10, (2, 400))
    yield "additive_2d", X2, np.maximum(0, X2[0] - 3) + 2 * np.maximum(0, 7 - X2[1]) + 0.01 * rng.normal(size=400)
    L = 64.0 * rng.integers(1, 129, 1500)                           # NW sequence lengths
    yield "nw_counter", L[None, :], 1e-3 * L**1.5 + 40 * np.log(L) + rng.normal(0, 5, 1500)
    X3 = np.stack([L, rng.integers(0, 3, 1500).astype(float), rng.uniform(0, 1, 1500)])
    yield "nw_3pred", X3, 1e-3 * L**1.5 * (1 + 0.3 * X3[1]) + rng.normal(0, 5, 1500)


@pytest.mark.parametrize("case", [c[0] for c in _mars_cases()])
def test_mars_parity(case):
    name, X, y = next(c for c in _mars_cases() if c[0] == case)
    mo = Ms.mars_fit(X, y)
    mg = bf.mars_fit(dev(X), dev(y))
    to = [(0, 0.0, 0) if t is None else t for t in mo["terms"]]
    assert mg["terms"] == to, (mg["terms"], to)
    scale = np.abs(y).max()
    fo, fg = Ms.mars_predict(mo, X), bf.mars_predict(mg, dev(X)).cpu().numpy()
    assert np.all(np.abs(fg - fo) <= 1e-9 * scale)
    tss = ((y - y.mean()) ** 2).sum()
    assert abs(mg["rss"] - mo["rss"]) <= 1e-9 * mo["rss"] + 1e-12 * tss
    assert abs(mg["rsq"] - mo["rsq"]) <= 1e-9
    assert abs(mg["gcv"] - mo["gcv"]) <= 1e-9 * mo["gcv"] + 1e-12 * tss / X.shape[1]
    # host-pointer path and new rows
    mh = bf.mars_fit(X, y)
    assert mh["terms"] == mg["terms"]
    Xn = X + 0.37
    assert np.allclose(bf.mars_predict(mg, Xn), Ms.mars_predict(mo, Xn), rtol=0, atol=1e-9 * scale)


def test_mars_edge_cases():
    rng = np.random.default_rng(2)
    # a constant predictor has no knots; the other carries the model
    x = rng.uniform(0, 5, 300)
    X = np.stack([np.full(300, 3.0), x])
    y = np.abs(x - 2.0) + 0.01 * rng.normal(size=300)
    mg, mo = bf.mars_fit(dev(X), dev(y)), Ms.mars_fit(X, y)
    assert mg["terms"] == [(0, 0.0, 0) if t is None else t for t in mo["terms"]]
    assert all(t[0] == 1 for t in mg["terms"][1:])
    # constant response: intercept only
    mc = bf.mars_fit(dev(X), dev(np.full(300, 7.5)))
    assert mc["terms"] == [(0, 0.0, 0)] and abs(mc["coef"][0] - 7.5) < 1e-12 and mc["rss"] <= 1e-20
    # two distinct values: no interior knot, intercept only
    X2 = np.array([[0.0, 1.0, 0.0, 1.0, 1.0]])
    m2 = bf.mars_fit(dev(X2), dev(np.array([1.0, 2.0, 1.0, 2.0, 2.0])))
    assert m2["terms"] == [(0, 0.0, 0)]
    # too many predictors for the default 31-term cap
    with pytest.raises(bf.BFError) as ei:
        bf.mars_fit(dev(rng.normal(size=(16, 50))), dev(rng.normal(size=50)))
    assert ei.value.code == -1


def test_glm_single_column_and_ragged_host():
    rng = np.random.default_rng(4)
    n = 1001
    Z = np.ones((1, n))
    Y = rng.normal(size=(3, n)) + np.array([[1.0], [2.0], [3.0]])
    g = bf.glm_gaussian(Z, Y)                       # intercept-only model, host pointers
    assert np.allclose(g["coef"][:, 0], Y.mean(axis=1), rtol=1e-13)
    assert np.allclose(g["deviance"], g["null_deviance"], rtol=1e-12)
