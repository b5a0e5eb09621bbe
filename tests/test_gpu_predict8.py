"""GPU parity of the compact-node prediction path (k_predict8, predict.cu).

k_predict8 decides x <= thr on floats and falls back to fp64 only when the
two round to the same float.  These cases stress exactly that
fallback (values above 2^24, where neighbouring integers share a float; query
values equal to thresholds and to their fp64 neighbours), single-node trees,
NaN queries, many tree blocks and ragged row counts, against the oracle
(S5: 1e-9 relative) and against the Node16 path (same leaves: 1e-12).
"""
from __future__ import annotations

import os

import numpy as np
import pytest

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():
    pytest.skip("no CUDA device", allow_module_level=True)

import paper_conf_ipps_madougouvln16_b200 as bf  # noqa: E402
from paper_conf_ipps_madougouvln16_b200 import synthetic as S  # noqa: E402
from oracle import oracle as O  # noqa: E402
from tests.helpers import rel_close  # noqa: E402

DEV = torch.device("cuda:0")


def dev(a):
    return torch.from_numpy(np.ascontiguousarray(a)).to(DEV)


def _predict(gf, Q, T, env=None):
    old = {k: os.environ.get(k) for k in (env or {})}
    try:
        for k, v in (env or {}).items():
            os.environ[k] = v
        ys, yh = gf.predict(dev(Q), ntree_total=T)
        return ys.cpu().numpy(), yh.cpu().numpy()
    finally:
        for k, v in old.items():
            if v is None:
                os.environ.pop(k, None)
            else:
                os.environ[k] = v


def _float_tie_data(n=3000, p=6, seed=5):
    rng = np.random.default_rng(seed)
    X = np.empty((p, n))
    X[0] = 2.0**30 + rng.integers(0, 40, n)            # neighbours share a float (ulp_f32 = 128)
    X[1] = 1e9 + rng.integers(0, 200, n) * 0.5
    X[2] = rng.integers(0, 50, n) * (1.0 + 2.0**-40)   # distinct in fp64, equal in fp32 per step
    X[3] = rng.normal(size=n)
    X[4] = -(2.0**26) - rng.integers(0, 30, n)
    X[5] = rng.integers(0, 3, n).astype(float)
    y = X[0] * 1e-9 + np.sin(X[3]) + 0.01 * rng.normal(size=n) + (X[2] > 20)
    return X, y


def _queries(X, gf, rng, m):
    """Training rows, thresholds themselves and their fp64 neighbours, and random mixes."""
    e = gf.export()
    thr = e["thr_or_value"][e["feature"] >= 0]
    feat = e["feature"][e["feature"] >= 0]
    p, n = X.shape
    Q = X[:, rng.integers(0, n, m)].copy()
    k = rng.integers(0, thr.size, m)
    which = rng.integers(0, 3, m)
    v = thr[k]
    v = np.where(which == 1, np.nextafter(v, np.inf), np.where(which == 2, np.nextafter(v, -np.inf), v))
    half = rng.random(m) < 0.5
    Q[feat[k][half], np.nonzero(half)[0]] = v[half]
    return Q


@pytest.mark.parametrize("mtry,ns", [(0, 5), (6, 1)])
def test_predict8_float_ties_vs_oracle_and_node16(mtry, ns):
    X, y = _float_tie_data()
    T = 24
    seed = 99 + ns
    of = O.fit(X, y, ntree=T, mtry=mtry, nodesize=ns, seed=seed, nthreads=4)
    gf = bf.fit(dev(X), dev(y), ntree=T, mtry=mtry, nodesize=ns, seed=seed)
    rng = np.random.default_rng(7)
    Q = _queries(X, gf, rng, 20011)  # ragged: not a multiple of the 128-row tile
    ys8, yh8 = _predict(gf, Q, T)
    ys16, _ = _predict(gf, Q, T, {"BF_PREDICT_NODE16": "1"})
    po = of.predict_sum(Q)
    assert rel_close(ys8, po, 1e-9)
    assert rel_close(yh8, po / T, 1e-9)
    assert rel_close(ys8, ys16, 1e-12)


def test_predict8_single_trees_exact_leaf():
    """One tree: the prediction IS a leaf value, so the two node formats must agree bit for bit."""
    X, y = _float_tie_data(seed=11)
    gf = bf.fit(dev(X), dev(y), ntree=1, nodesize=1, seed=3)
    Q = _queries(X, gf, np.random.default_rng(3), 5000)
    a, _ = _predict(gf, Q, 1)
    b, _ = _predict(gf, Q, 1, {"BF_PREDICT_NODE16": "1"})
    assert np.array_equal(a, b)


def test_predict8_single_node_trees_mixed_with_deep_trees():
    X, y = S.small_random(400, 5, seed=1, kind="mixed")
    deep = bf.fit(dev(X), dev(y), ntree=5, seed=1).export()
    stump = bf.fit(dev(X[:, :4]), dev(y[:4]), ntree=3, seed=2).export()  # n = 4 <= nodesize: single leaves
    assert np.all(stump["feature"] == -1)
    # interleave: stump, deep, stump, deep ... through bf_forest_import
    trees = []
    for i in range(5):
        for src, j in ((stump, min(i, 2)), (deep, i)):
            lo, hi = src["tree_off"][j], src["tree_off"][j + 1]
            trees.append({k: src[k][lo:hi] for k in ("feature", "left", "thr_or_value", "count", "value", "drss")})
    arrays = {k: np.concatenate([t[k] for t in trees]) for k in trees[0]}
    arrays["tree_off"] = np.concatenate([[0], np.cumsum([t["feature"].size for t in trees])]).astype(np.int64)
    info = deep["info"]
    info.tree_begin, info.tree_end, info.ntree_total = 0, len(trees), len(trees)
    info.total_nodes = int(arrays["tree_off"][-1])
    f = bf.forest_import(arrays, info)
    Q = S.gen_query(X, 3001)
    a, _ = _predict(f, Q, len(trees))
    b, _ = _predict(f, Q, len(trees), {"BF_PREDICT_NODE16": "1"})
    assert rel_close(a, b, 1e-12)
    # host reference: walk the exported arrays
    ref = np.zeros(Q.shape[1])
    for t in trees:
        for r in range(Q.shape[1]):
            k = 0
            while t["feature"][k] >= 0:
                k = t["left"][k] + (0 if Q[t["feature"][k], r] <= t["thr_or_value"][k] else 1)
            ref[r] += t["thr_or_value"][k]
    assert rel_close(a, ref, 1e-12)


def test_predict8_nan_queries_go_right_like_node16():
    X, y = S.small_random(600, 4, seed=4, kind="cont")
    gf = bf.fit(dev(X), dev(y), ntree=6, seed=4)
    Q = S.gen_query(X, 777)
    Q[1, ::3] = np.nan
    Q[2, ::5] = np.inf
    Q[0, ::7] = -np.inf
    a, _ = _predict(gf, Q, 6)
    b, _ = _predict(gf, Q, 6, {"BF_PREDICT_NODE16": "1"})
    assert rel_close(a, b, 1e-12)


@pytest.mark.parametrize("block", ["4096", "100000"])
def test_predict8_many_tree_blocks(block):
    X, y, c = S.dataset("C1")
    T = 37
    of = O.fit(X, y, ntree=T, seed=S.FOREST_SEED + 2, nthreads=4)
    gf = bf.fit(dev(X), dev(y), ntree=T, seed=S.FOREST_SEED + 2)
    Q = S.gen_query(X, 1000)
    a, ah = _predict(gf, Q, T, {"BF_PREDICT_BLOCK_BYTES": block})
    po = of.predict_sum(Q)
    assert rel_close(a, po, 1e-9)
    assert rel_close(ah, po / T, 1e-9)


@pytest.mark.parametrize("m", [0, 1, 127, 129])
def test_predict8_tiny_row_counts(m):
    X, y = S.small_random(300, 3, seed=8, kind="int")
    gf = bf.fit(dev(X), dev(y), ntree=9, seed=8)
    of = O.fit(X, y, ntree=9, seed=8)
    Q = S.gen_query(X, max(m, 1))[:, :m]
    a, _ = _predict(gf, np.ascontiguousarray(Q), 9)
    assert a.shape == (m,)
    if m:
        assert rel_close(a, of.predict_sum(np.ascontiguousarray(Q)), 1e-9)


@pytest.mark.parametrize("node16", [False, True])
def test_importance_float_ties_vs_oracle(node16):
    """OOB importance walks (original and permuted) on the compact nodes take the fp64 decision on float
    ties: slots, OOB sums and counts agree with the oracle (S6-S7 tolerances) on tie-heavy data."""
    X, y = _float_tie_data(n=2000, seed=21)
    T = 12
    of = O.fit(X, y, ntree=T, seed=5, nthreads=4)
    gf = bf.fit(dev(X), dev(y), ntree=T, seed=5)
    env = {"BF_PREDICT_NODE16": "1"} if node16 else {}
    old = {k: os.environ.get(k) for k in env}
    try:
        os.environ.update(env)
        r = gf.oob_importance(dev(X), dev(y))
    finally:
        for k, v in old.items():
            if v is None:
                os.environ.pop(k, None)
    ro = of.oob_importance(X, y)
    assert np.array_equal(r["nout_t"].cpu().numpy(), ro["nout_t"])
    assert np.array_equal(r["oob_cnt"].cpu().numpy(), ro["oob_cnt"])
    assert rel_close(r["oob_sum"].cpu().numpy(), ro["oob_sum"], 1e-9)
    assert rel_close(r["e_t"].cpu().numpy(), ro["e_t"], 1e-9)
    ds = ro["d_slots"]
    assert rel_close(r["d_slots"].cpu().numpy(), ds, 1e-6, atol_scale=1e-9)


def test_wide_forest_uses_node16_path_and_matches_oracle():
    """p = 300 > 256: the compact layout cannot hold the feature index, so predict and importance take the
    Node16 kernels automatically; both still agree with the oracle."""
    rng = np.random.default_rng(30)
    n, p, T = 400, 300, 6
    X = rng.normal(size=(p, n))
    y = X[7] + 0.5 * X[280] ** 2 + 0.1 * rng.normal(size=n)
    of = O.fit(X, y, ntree=T, seed=4, nthreads=4)
    gf = bf.fit(dev(X), dev(y), ntree=T, seed=4)
    Q = S.gen_query(X, 999)
    ys, _ = _predict(gf, Q, T)
    assert rel_close(ys, of.predict_sum(Q), 1e-9)
    r = gf.oob_importance(dev(X), dev(y))
    ro = of.oob_importance(X, y)
    assert np.array_equal(r["oob_cnt"].cpu().numpy(), ro["oob_cnt"])
    assert rel_close(r["d_slots"].cpu().numpy(), ro["d_slots"], 1e-6, atol_scale=1e-9)
