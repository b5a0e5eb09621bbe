"""GPU parity of the two-level 32-byte group walks (k_predict32, predict.cu; k_importance32, importance.cu).

A G32 group holds an internal node at even depth and its two children; one 256-bit load decides two levels
and the grandchild slot is loaded next.  The walk must take exactly the S5 path (P:95 step 3):
the same float-then-fp64 comparison as the Node8 walk, so on one forest the two agree to 1e-12 (leaf sums in
the same tree order) and both agree with the oracle to 1e-9 relative.  The cases stress the fp64 tie fallback
at both levels of a group (its node ids come from the group), single-node trees (root slot is a leaf), leaf
children and leaf grandchildren, many tree blocks, NaN / inf queries and ragged row counts.
"""
from __future__ import annotations

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
from tests.test_gpu_predict8 import _float_tie_data, _predict, _queries, dev  # noqa: E402

G32 = {"BF_PREDICT_V": "3"}
N8 = {"BF_PREDICT_V": "2"}


@pytest.mark.parametrize("mtry,ns", [(0, 5), (6, 1), (0, 2)])
def test_predict32_float_ties_vs_oracle_and_node8(mtry, ns):
    X, y = _float_tie_data()
    T = 24
    seed = 199 + ns
    of = O.fit(X, y, ntree=T, mtry=mtry, nodesize=ns, seed=seed, nthreads=4)
    gf = bf.fit(dev(X), dev(y), ntree=T, mtry=mtry, nodesize=ns, seed=seed)
    Q = _queries(X, gf, np.random.default_rng(17), 20011)
    a, ah = _predict(gf, Q, T, G32)
    b, _ = _predict(gf, Q, T, N8)
    c, _ = _predict(gf, Q, T, {"BF_PREDICT_NODE16": "1"})
    po = of.predict_sum(Q)
    assert rel_close(a, po, 1e-9)
    assert rel_close(ah, po / T, 1e-9)
    assert rel_close(a, b, 1e-12)
    assert rel_close(a, c, 1e-12)


@pytest.mark.parametrize("seed", [3, 4, 5])
def test_predict32_single_tree_is_a_leaf_value(seed):
    """One tree: the prediction IS a leaf value (odd-depth leaves come from the group, even-depth leaves from
    their own slot), so G32 and Node16 must agree bit for bit."""
    X, y = _float_tie_data(seed=seed + 10)
    gf = bf.fit(dev(X), dev(y), ntree=1, nodesize=1 + seed % 3, seed=seed)
    Q = _queries(X, gf, np.random.default_rng(seed), 5000)
    a, _ = _predict(gf, Q, 1, G32)
    b, _ = _predict(gf, Q, 1, {"BF_PREDICT_NODE16": "1"})
    assert np.array_equal(a, b)


def test_predict32_single_node_and_two_level_trees_mixed_with_deep_trees():
    X, y = S.small_random(400, 5, seed=1, kind="mixed")
    deep = bf.fit(dev(X), dev(y), ntree=5, seed=1).export()
    stump = bf.fit(dev(X[:, :4]), dev(y[:4]), ntree=3, seed=2).export()  # single leaves
    assert np.all(stump["feature"] == -1)
    trees = []
    for i in range(5):
        for src, j in ((stump, min(i, 2)), (deep, i)):
            lo, hi = src["tree_off"][j], src["tree_off"][j + 1]
            trees.append({k: src[k][lo:hi] for k in ("feature", "left", "thr_or_value", "count", "value", "drss")})
    # a one-split tree: root internal, both children leaves (no grandchildren)
    t0 = trees[1]
    k = int(np.nonzero(t0["feature"] >= 0)[0][0])
    one = {key: t0[key][:3].copy() for key in t0}
    one["feature"][:] = [t0["feature"][k], -1, -1]
    one["left"][:] = [1, -1, -1]
    one["thr_or_value"][:] = [t0["thr_or_value"][k], -1.5, 2.5]
    trees.append(one)
    arrays = {k: np.concatenate([t[k] for t in trees]) for k in trees[0]}
    arrays["tree_off"] = np.concatenate([[0], np.cumsum([t["feature"].size for t in trees])]).astype(np.int64)
    info = deep["info"]
    info.tree_begin, info.tree_end, info.ntree_total = 0, len(trees), len(trees)
    info.total_nodes = int(arrays["tree_off"][-1])
    f = bf.forest_import(arrays, info)
    Q = S.gen_query(X, 3001)
    a, _ = _predict(f, Q, len(trees), G32)
    ref = np.zeros(Q.shape[1])
    for t in trees:
        for r in range(Q.shape[1]):
            k = 0
            while t["feature"][k] >= 0:
                k = t["left"][k] + (0 if Q[t["feature"][k], r] <= t["thr_or_value"][k] else 1)
            ref[r] += t["thr_or_value"][k]
    assert rel_close(a, ref, 1e-12)


def test_predict32_nan_and_inf_queries_like_node16():
    X, y = S.small_random(600, 4, seed=4, kind="cont")
    gf = bf.fit(dev(X), dev(y), ntree=6, seed=4)
    Q = S.gen_query(X, 777)
    Q[1, ::3] = np.nan
    Q[2, ::5] = np.inf
    Q[0, ::7] = -np.inf
    a, _ = _predict(gf, Q, 6, G32)
    b, _ = _predict(gf, Q, 6, {"BF_PREDICT_NODE16": "1"})
    assert rel_close(a, b, 1e-12)


@pytest.mark.parametrize("block", ["4096", "100000"])
def test_predict32_many_tree_blocks(block):
    X, y, c = S.dataset("C1")
    T = 37
    of = O.fit(X, y, ntree=T, seed=S.FOREST_SEED + 2, nthreads=4)
    gf = bf.fit(dev(X), dev(y), ntree=T, seed=S.FOREST_SEED + 2)
    Q = S.gen_query(X, 1000)
    a, ah = _predict(gf, Q, T, dict(G32, BF_PREDICT_BLOCK_BYTES=block))
    po = of.predict_sum(Q)
    assert rel_close(a, po, 1e-9)
    assert rel_close(ah, po / T, 1e-9)


@pytest.mark.parametrize("m", [1, 127, 129])
def test_predict32_tiny_row_counts(m):
    X, y = S.small_random(300, 3, seed=8, kind="int")
    gf = bf.fit(dev(X), dev(y), ntree=9, seed=8)
    of = O.fit(X, y, ntree=9, seed=8)
    Q = np.ascontiguousarray(S.gen_query(X, m))
    a, _ = _predict(gf, Q, 9, G32)
    assert rel_close(a, of.predict_sum(Q), 1e-9)


@pytest.mark.parametrize("cfg", ["C2", "C3"])
def test_predict32_configs_vs_oracle(cfg):
    X, y, c = S.dataset(cfg)
    T = 40
    of = O.fit(X, y, ntree=T, seed=S.FOREST_SEED + 5, nthreads=8)
    gf = bf.fit(dev(X), dev(y), ntree=T, seed=S.FOREST_SEED + 5)
    Q = S.gen_query(X, 4099)
    a, _ = _predict(gf, Q, T, G32)
    assert rel_close(a, of.predict_sum(Q), 1e-9)


@pytest.mark.parametrize("env", [{}, {"BF_PREDICT_V": "2"}])
@pytest.mark.parametrize("mtry,ns", [(0, 5), (6, 1)])
def test_importance32_float_ties_vs_oracle(env, mtry, ns):
    """OOB importance on the G32 groups (default for p <= 64; BF_PREDICT_V=2: the Node8 walks): a permuted walk
    starts at a group's node or at its chosen child, the fp64 tie decisions use the permuted fp64 value; the
    slots, OOB sums and counts agree with the oracle (S6-S7 tolerances) on tie-heavy data."""
    import os
    X, y = _float_tie_data(n=2000, seed=21 + ns)
    T = 12
    of = O.fit(X, y, ntree=T, mtry=mtry, nodesize=ns, seed=5, nthreads=4)
    gf = bf.fit(dev(X), dev(y), ntree=T, mtry=mtry, nodesize=ns, seed=5)
    old = {k: os.environ.get(k) for k in env}
    try:
        os.environ.update(env)
        r = gf.oob_importance(dev(X), dev(y))
    finally:
        for k, v in old.items():
            if v is None:
                os.environ.pop(k, None)
            else:
                os.environ[k] = v
    ro = of.oob_importance(X, y)
    assert np.array_equal(r["nout_t"].cpu().numpy(), ro["nout_t"])
    assert np.array_equal(r["oob_cnt"].cpu().numpy(), ro["oob_cnt"])
    assert rel_close(r["oob_sum"].cpu().numpy(), ro["oob_sum"], 1e-9)
    assert rel_close(r["e_t"].cpu().numpy(), ro["e_t"], 1e-9)
    assert rel_close(r["d_slots"].cpu().numpy(), ro["d_slots"], 1e-6, atol_scale=1e-9)
    assert np.all(r["d_slots"].cpu().numpy()[ro["d_slots"] == 0.0] == 0.0)
