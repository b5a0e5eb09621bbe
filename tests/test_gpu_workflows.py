"""GPU parity of the composed workflows (workflows.py; SURVEY 8(f) NEXT-3,
NEXT-4) against the same composition of the oracle: retained predictors,
counter models, modelled test rows, predicted times and the importance-ranking
similarity of per-generation forests."""
from __future__ import annotations

import math

import numpy as np
import pytest

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():
    pytest.skip("no CUDA device", allow_module_level=True)

import paper_conf_ipps_madougouvln16_b200 as bf  # noqa: E402
from paper_conf_ipps_madougouvln16_b200 import synthetic as S  # noqa: E402
from paper_conf_ipps_madougouvln16_b200 import workflows as W  # noqa: E402
from oracle import oracle as O  # noqa: E402
from oracle import pca as OP  # noqa: E402
from oracle import scaling as Sc  # noqa: E402
from tests.helpers import rel_close  # noqa: E402

DEV = torch.device("cuda:0")


def dev(a):
    return torch.from_numpy(np.ascontiguousarray(a)).to(DEV)


def _oracle_inc_mse(X, y, T, seed):
    of = O.fit(X, y, ntree=T, seed=seed, nthreads=8)
    r = of.oob_importance(X, y)
    return of, O.importance_finalize(r["d_slots"], r["npur_slots"], r["oob_sum"], r["oob_cnt"], y)["inc_mse"]


def test_problem_scaling_mm_matches_oracle_composition():
    X, y, c = S.dataset("C2")
    size_row = X.shape[0] - 1                                   # N (gen_mm: last predictor)
    sizes = np.unique(X[size_row])
    unseen = sizes[2::5]                                        # every 5th size is never trained on
    te_mask = np.isin(X[size_row], unseen)
    tr, te = np.nonzero(~te_mask)[0], np.nonzero(te_mask)[0]
    T, seed = 40, 77
    r = W.problem_scaling(dev(X), dev(y), size_row, dev(tr), dev(te), top=6, ntree=T, seed=seed)
    # retained set = the oracle forest's %IncMSE ranking
    _, imp = _oracle_inc_mse(X[:, tr], y[tr], T, seed)
    assert r["keep"] == list(np.argsort(-imp, kind="stable")[:6])
    # counter models on the same design
    keep_c = [j for j in r["keep"] if j != size_row]
    Ztr = W.log_size_design(dev(X[size_row, tr])).cpu().numpy()
    co, do, no = Sc.glm_gaussian(Ztr.T, X[keep_c][:, tr].T)
    scale = np.abs(X[keep_c][:, tr]).max(axis=1, keepdims=True)
    assert np.all(np.abs(r["coef"].cpu().numpy() @ Ztr - co.T @ Ztr) <= 1e-10 * scale)
    assert np.all(np.abs(r["deviance"].cpu().numpy() - do) <= 1e-8 * do + 1e-12 * no)
    # predicted times: the oracle forest on the retained set, walked on the GPU's modelled rows
    Xh = r["X_model"].cpu().numpy()
    ofk = O.fit(np.ascontiguousarray(X[r["keep"]][:, tr]), y[tr], ntree=T, seed=seed + 1, nthreads=8)
    assert rel_close(r["yhat"].cpu().numpy(), ofk.predict_sum(Xh) / T, 1e-9)
    assert r["test_explained"] > 0.5


def test_hardware_scaling_nw_matches_oracle_composition():
    Xc, L, M, y = S.gen_nw(4096)
    gen = np.array([{13: 1, 15: 0, 16: 2}[int(v)] for v in M[2]])  # SM count identifies the generation
    T, seed = 30, 5
    r = W.hardware_scaling(dev(Xc), dev(L), dev(M), dev(y), dev(gen), (0, 1), 2, ntree=T, seed=seed)
    po = OP.pca(Xc, scale=True)
    assert r["k"] == OP.n_components(po["sdev"])
    R = r["inputs"].cpu().numpy()
    tr, te = np.nonzero(gen != 2)[0], np.nonzero(gen == 2)[0]
    of = O.fit(np.ascontiguousarray(R[:, tr]), y[tr], ntree=T, seed=seed, nthreads=8)
    assert rel_close(r["yhat"].cpu().numpy(), of.predict_sum(np.ascontiguousarray(R[:, te])) / T, 1e-9)
    imps = []
    for g in (0, 1):
        ig = np.nonzero(gen == g)[0]
        _, imp = _oracle_inc_mse(np.ascontiguousarray(R[:, ig]), y[ig], T, seed + 1 + g)
        assert np.array_equal(np.argsort(-imp, kind="stable"),
                              np.argsort(-r["inc_mse_per_gen"][g].cpu().numpy(), kind="stable"))
        imps.append(imp)
    rho, tau = r["similarity"][(0, 1)]
    assert math.isclose(rho, Sc.spearman(imps[0], imps[1]), rel_tol=1e-9, abs_tol=1e-12)
    assert math.isclose(tau, Sc.kendall_tau_b(imps[0], imps[1]), rel_tol=1e-9, abs_tol=1e-12)


def test_problem_scaling_nw_with_mars_matches_oracle_composition():
    from oracle import mars as Ms
    Xc, L, M, y = S.gen_nw(6000)
    g0 = M[2] == 15                                              # one GPU (GTX480 rows)
    X = np.ascontiguousarray(np.concatenate([Xc[:, g0], L[None, g0]], axis=0))
    yy = y[g0]
    size_row = X.shape[0] - 1
    unseen = np.unique(X[size_row])[3::7]
    te_mask = np.isin(X[size_row], unseen)
    tr, te = np.nonzero(~te_mask)[0], np.nonzero(te_mask)[0]
    T, seed = 30, 9
    r = W.problem_scaling(dev(X), dev(yy), size_row, dev(tr), dev(te), top=6, ntree=T, seed=seed,
                          counter_model="mars")
    _, imp = _oracle_inc_mse(X[:, tr], yy[tr], T, seed)
    assert r["keep"] == list(np.argsort(-imp, kind="stable")[:6])
    keep_c = [j for j in r["keep"] if j != size_row]
    for j, mg in zip(keep_c, r["models"]["mars"]):
        mo = Ms.mars_fit(X[size_row, tr][None, :], X[j, tr])
        assert mg["terms"] == [(0, 0.0, 0) if t is None else t for t in mo["terms"]]
    Xh = r["X_model"].cpu().numpy()
    ofk = O.fit(np.ascontiguousarray(X[r["keep"]][:, tr]), yy[tr], ntree=T, seed=seed + 1, nthreads=8)
    assert rel_close(r["yhat"].cpu().numpy(), ofk.predict_sum(Xh) / T, 1e-9)


def test_log_size_design_and_prediction_error_vs_oracle():
    """The workflow statistics on the device (bf_log_size_design, bf_prediction_error) against the oracle's
    plain definitions, on the paper's size grids and on random data (device and host pointers)."""
    rng = np.random.default_rng(3)
    for s in (2.0 ** np.arange(5, 12), np.arange(64, 8193, 64, dtype=np.float64), rng.uniform(1, 1e6, 999)):
        Zg = bf.log_size_design(dev(s)).cpu().numpy()
        Zo = Sc.log_size_design(s)
        assert np.allclose(Zg, Zo, rtol=1e-13, atol=1e-13)
        assert np.allclose(bf.log_size_design(np.ascontiguousarray(s)), Zo, rtol=1e-13, atol=1e-13)
    y = rng.normal(size=5000)
    yh = y + 0.1 * rng.normal(size=5000)
    mg, eg = bf.prediction_error(dev(yh), dev(y))
    mo, eo = Sc.prediction_error(yh, y)
    assert math.isclose(mg, mo, rel_tol=1e-12) and math.isclose(eg, eo, rel_tol=1e-12)
    assert math.isnan(bf.prediction_error(dev(np.ones(4)), dev(np.full(4, 2.0)))[1])
