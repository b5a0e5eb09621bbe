"""Pins of the CPU oracle against what the paper and mathematics fix.

Nothing here compares the oracle with itself: every expected value comes
from a published test vector, exact rational arithmetic, a closed form, an
invariant, a library routine (sklearn / numpy.linalg) or brute force.
Cites: P:n = PAPER.md line n, S1..S9 = DESIGN.md section 2.
"""
from __future__ import annotations

import math
import os
import random
from fractions import Fraction

import numpy as np
import pytest

from oracle import oracle as O
from tests.brute import brute_tree, rss

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


# ---------------------------------------------------------------- S1 Philox
def test_philox_known_answers():
    """Random123 published KAT vectors (tests/golden/philox_kat.txt)."""
    rows = [l.split() for l in open(os.path.join(GOLDEN, "philox_kat.txt")) if l.strip() and not l.startswith("#")]
    assert len(rows) == 3
    for r in rows:
        v = [int(x, 16) for x in r]
        assert O.philox(v[0:4], v[4:6]) == v[6:10]


def test_mulhi64_is_floor_of_product():
    rng = random.Random(1)
    for _ in range(2000):
        u = rng.getrandbits(64)
        r = rng.randrange(1, 1 << 40)
        got = O.mulhi64(u, r)
        assert got == (u * r) >> 64
        assert 0 <= got < r


def test_int128_to_double_correctly_rounded():
    """Python float(int) is correctly rounded (round-half-even)."""
    rng = random.Random(2)
    cases = [0, 1, -1, (1 << 53) + 1, -((1 << 53) + 1), ((1 << 53) + 1) << 40, ((1 << 54) + 3) << 30,
             (1 << 127) - 1, -(1 << 127), ((1 << 53) + 1) << 70, (((1 << 53) + 1) << 20) + 1]
    for _ in range(3000):
        b = rng.randrange(1, 127)
        v = rng.getrandbits(b)
        if rng.random() < 0.3:  # near-halfway: 54 significant bits + tail
            v = ((rng.getrandbits(53) | (1 << 53)) * 2 + 1) << rng.randrange(0, 60)
            v &= (1 << 126) - 1
        cases.append(-v if rng.random() < 0.5 else v)
    for v in cases:
        assert O.i128_to_double(v) == float(v), v


# ---------------------------------------------------------------- S2 fixed point
def test_fixed_point_exact_for_small_integers():
    y = np.array([-5, -3, 0, 1, 4, 4, 2], np.float64)
    yq, q = O.fixed_point(y)
    c = 0.5 * y.min() + 0.5 * y.max()
    # y - c has few bits: the scaling by 2^q is exact, so y_q is an exact affine image of y
    assert np.all(np.ldexp(yq.astype(np.float64), -q) + c == y)
    s = int(len(y)).bit_length()
    assert np.abs(yq).max() <= 1 << (62 - s)


@pytest.mark.parametrize("n", [1, 7, 256, 4096, 100000])
def test_fixed_point_bounds(n):
    rng = np.random.default_rng(n)
    y = rng.lognormal(0, 3, n) * (1 if n % 2 else -1)
    yq, q = O.fixed_point(y)
    s = int(n).bit_length()
    if n == 1:
        assert np.all(yq == 0)
        return
    c = 0.5 * y.min() + 0.5 * y.max()
    R = np.abs(y - c).max()
    # q chosen so that R * 2^q in [2^(61-s), 2^(62-s))
    assert 2.0 ** (61 - s) <= R * 2.0 ** q < 2.0 ** (62 - s)
    assert np.abs(yq).max() <= 1 << (62 - s)
    # sum of N_s values cannot overflow int64
    assert n * int(np.abs(yq).max()) < 1 << 63
    # rounding error at most half a unit of 2^-q
    err = np.abs(np.ldexp(yq.astype(np.float64), -q) - (y - c))
    assert np.all(err <= 2.0 ** (-q - 1) * (1 + 1e-12))


# ---------------------------------------------------------------- S3 bootstrap
@pytest.mark.parametrize("n", [256, 4096, 100000])
def test_bootstrap_statistics(n):
    ws = [O.bootstrap(0xBF10_0000, t, n) for t in range(8)]
    frac = []
    for w in ws:
        assert int(w.sum()) == n               # sum of multiplicities = N_s exactly
        assert w.min() >= 0
        frac.append((w > 0).mean())
    expect = 1 - (1 - 1 / n) ** n               # E[distinct]/n
    sd = math.sqrt(expect * (1 - expect) / n)   # binomial-ish spread bound
    assert abs(np.mean(frac) - expect) < 6 * sd / math.sqrt(8) + 2e-3
    # multiplicity histogram vs Binomial(N_s, 1/n) (chi-square, k = 0..4, tail pooled)
    w = np.concatenate(ws)
    obs = np.array([(w == k).sum() for k in range(4)] + [(w >= 4).sum()], np.float64)
    pk = [math.comb(n, k) * (1 / n) ** k * (1 - 1 / n) ** (n - k) for k in range(4)]
    exp = np.array(pk + [1 - sum(pk)]) * len(w)
    chi2 = ((obs - exp) ** 2 / exp).sum()
    assert chi2 < 30.0  # 4 dof; p ~ 5e-6


def test_bootstrap_trees_differ_and_replace0():
    a = O.bootstrap(7, 0, 1000)
    b = O.bootstrap(7, 1, 1000)
    assert not np.array_equal(a, b)
    assert np.all(O.bootstrap(7, 3, 50, replace=0) == 1)


# ---------------------------------------------------------------- S3 mtry
def test_mtry_draw_is_uniform_subset():
    p, mtry = 20, 6
    counts = np.zeros(p)
    key = 0
    for i in range(20000):
        key = O.child_key(5, 3, key, i & 1)
        f = O.draw_mtry(5, 3, key, p, mtry)
        assert len(set(f.tolist())) == mtry and f.min() >= 0 and f.max() < p
        counts[f] += 1
    exp = 20000 * mtry / p
    chi2 = ((counts - exp) ** 2 / exp).sum()
    assert chi2 < 60  # 19 dof
    assert sorted(O.draw_mtry(1, 2, 3, 9, 9).tolist()) == list(range(9))  # mtry = p: a permutation


def test_child_keys_distinct():
    ks = set()
    frontier = [0]
    for _ in range(12):
        nxt = []
        for k in frontier:
            for s in (0, 1):
                c = O.child_key(11, 4, k, s)
                nxt.append(c)
                ks.add(c)
        frontier = nxt
    assert len(ks) == 2 ** 13 - 2


# ---------------------------------------------------------------- S7 Feistel
@pytest.mark.parametrize("n_o", list(range(1, 140)) + [255, 256, 257, 1000, 4097])
def test_feistel_is_bijection(n_o):
    img = [O.perm(9, 2, 5, n_o, a) for a in range(n_o)]
    assert sorted(img) == list(range(n_o))


def test_feistel_not_identity_and_spread():
    n_o = 1000
    img0 = [O.perm(9, t, 0, n_o, 0) for t in range(400)]
    assert len(set(img0)) > 300  # pi(0) spreads over [0, n_o)
    assert sum(O.perm(9, 1, 1, n_o, a) == a for a in range(n_o)) < 20


# ---------------------------------------------------------------- S4 tree growth vs exact rationals
def _oracle_tree(X, y, **kw):
    F = O.fit(X, y, ntree=1, **kw)
    return F, F.tree(0)


def _compare_to_brute(X, y, seed, nodesize, mtry):
    p, n = X.shape
    F, tr = _oracle_tree(X, y, seed=seed, nodesize=nodesize, mtry=mtry)
    w = O.bootstrap(seed, 0, n)
    draw = (lambda k: O.draw_mtry(seed, 0, k, p, mtry)) if mtry < p else None
    ck = lambda k, s: O.child_key(seed, 0, k, s)
    bt = brute_tree([list(c) for c in X], list(y), list(w), nodesize, draw=draw, child_key=ck)
    assert len(bt) == len(tr["feature"])
    for k, nd in enumerate(bt):
        assert tr["feature"][k] == nd["feature"], (k, nd)
        assert tr["count"][k] == nd["count"]
        assert tr["value"][k] == pytest.approx(float(nd["value"]), rel=1e-13, abs=1e-13)
        if nd["feature"] >= 0:
            assert tr["left"][k] == nd["left"]
            assert nd["a"] <= tr["thr"][k] < nd["b"]
            assert tr["drss"][k] == pytest.approx(float(nd["drss"]), rel=1e-9)


def test_split_search_vs_exact_rational_bruteforce_mtry_eq_p():
    rng = np.random.default_rng(3)
    for case in range(300):
        n = int(rng.integers(2, 13))
        p = int(rng.integers(1, 5))
        X = rng.integers(0, 5, (p, n)).astype(np.float64)   # many ties
        y = rng.integers(-5, 6, n).astype(np.float64)        # integer y: y_q exact affine image
        _compare_to_brute(X, y, seed=case, nodesize=int(rng.integers(1, 4)), mtry=p)


def test_split_search_vs_exact_rational_bruteforce_mtry_lt_p():
    rng = np.random.default_rng(4)
    for case in range(200):
        n = int(rng.integers(4, 16))
        p = int(rng.integers(2, 6))
        X = rng.integers(0, 6, (p, n)).astype(np.float64)
        y = rng.integers(-9, 10, n).astype(np.float64)
        _compare_to_brute(X, y, seed=1000 + case, nodesize=1, mtry=int(rng.integers(1, p)))


# ---------------------------------------------------------------- closed forms
def test_single_leaf_when_nodesize_ge_sample():
    X, y = np.random.default_rng(0).normal(size=(3, 40)), np.random.default_rng(1).normal(size=40)
    F = O.fit(X, y, ntree=3, nodesize=40, seed=2)
    for i in range(3):
        tr = F.tree(i)
        w = O.bootstrap(2, i, 40)
        assert len(tr["feature"]) == 1 and tr["feature"][0] == -1
        assert tr["value"][0] == pytest.approx(float(np.dot(w, y) / w.sum()), rel=1e-14)
    assert np.allclose(F.predict_sum(X) / 3, np.mean([F.tree(i)["value"][0] for i in range(3)]), rtol=1e-14)


def test_replace0_leaf_is_mean_and_constant_cases():
    rng = np.random.default_rng(5)
    X, y = rng.normal(size=(2, 30)), rng.normal(size=30)
    F = O.fit(X, y, ntree=1, nodesize=30, replace=0)
    assert F.tree(0)["value"][0] == pytest.approx(y.mean(), rel=1e-14)
    F = O.fit(X, np.full(30, 3.25), ntree=2, nodesize=1)          # constant y -> one leaf, value exact
    assert len(F.tree(1)["feature"]) == 1 and F.tree(1)["value"][0] == 3.25
    F = O.fit(np.ones((3, 30)), y, ntree=2, nodesize=1)           # constant X -> one leaf
    assert len(F.tree(0)["feature"]) == 1


def test_perfect_fit_nodesize1_distinct_columns():
    """Theorem: nodesize = 1 and all columns with distinct values
    -> every tree reproduces its in-bag responses exactly."""
    rng = np.random.default_rng(6)
    n, p = 200, 6
    X = np.stack([rng.permutation(n).astype(np.float64) for _ in range(p)])
    y = rng.integers(-1000, 1000, n).astype(np.float64)
    F = O.fit(X, y, ntree=4, nodesize=1, seed=9)
    for i in range(4):
        w = O.bootstrap(9, i, n)
        one = _walk_all(F.tree(i), X)
        inb = w > 0
        assert np.array_equal(one[inb], y[inb])


def _walk_all(tr, X):
    out = np.empty(X.shape[1])
    for r in range(X.shape[1]):
        k = 0
        while tr["feature"][k] >= 0:
            k = tr["left"][k] if X[tr["feature"][k], r] <= tr["thr"][k] else tr["left"][k] + 1
        out[r] = tr["value"][k]
    return out


# ---------------------------------------------------------------- invariants
def test_tree_invariants_counts_thresholds_telescoping():
    from paper_conf_ipps_madougouvln16_b200 import synthetic as S
    X, y = S.gen_reduction()
    p, n = X.shape
    seed = 0xBF10_0001
    F = O.fit(X, y, ntree=5, seed=seed)
    for i in range(5):
        tr = F.tree(i)
        w = O.bootstrap(seed, i, n)
        nn = len(tr["feature"])
        rows = {0: [r for r in range(n) if w[r] > 0]}
        for k in range(nn):  # BFS: parents before children
            R = rows[k]
            assert tr["count"][k] == sum(w[r] for r in R)
            if tr["feature"][k] >= 0:
                f, thr, l = tr["feature"][k], tr["thr"][k], tr["left"][k]
                L = [r for r in R if X[f, r] <= thr]
                Rr = [r for r in R if X[f, r] > thr]
                assert L and Rr
                assert max(X[f, r] for r in L) <= thr < min(X[f, r] for r in Rr)
                rows[l], rows[l + 1] = L, Rr
                assert tr["count"][l] + tr["count"][l + 1] == tr["count"][k]
                assert l > k
            else:
                assert tr["count"][k] <= 5 or len(set(y[R])) >= 1
        # RSS_root = sum(drss) + sum(RSS leaves)  (fp64 vs exact rationals)
        root = float(rss(rows[0], w, y))
        leaves = sum(float(rss(rows[k], w, y)) for k in range(nn) if tr["feature"][k] < 0)
        assert tr["drss"].sum() + leaves == pytest.approx(root, rel=1e-9)


def test_metamorphic_monotone_transform_and_y_scaling():
    rng = np.random.default_rng(7)
    n, p = 300, 5
    X = rng.normal(size=(p, n))
    y = rng.normal(size=n)
    F1 = O.fit(X, y, ntree=3, seed=1)
    X2 = X.copy()
    X2[2] = np.exp(X2[2]) * 3 + 1              # strictly increasing
    F2 = O.fit(X2, y, ntree=3, seed=1)
    F3 = O.fit(X, y * 8.0, ntree=3, seed=1)     # y * 2^3
    for i in range(3):
        a, b, c = F1.tree(i), F2.tree(i), F3.tree(i)
        assert np.array_equal(a["feature"], b["feature"]) and np.array_equal(a["left"], b["left"])
        assert np.array_equal(a["count"], b["count"])
        assert np.array_equal(a["feature"], c["feature"]) and np.array_equal(a["thr"], c["thr"])
        assert np.array_equal(c["value"], a["value"] * 8.0)
        assert np.array_equal(c["drss"], a["drss"] * 64.0)
    assert F3.q == F1.q - 3


def test_whole_tree_vs_sklearn():
    """sklearn DecisionTreeRegressor on the materialised bootstrap sample,
    max_features=None (= mtry = p), min_samples_split = nodesize + 1.
    Preconditions: integer-gap x, distinct gains."""
    sk = pytest.importorskip("sklearn.tree")
    rng = np.random.default_rng(8)
    for case in range(6):
        n, p = 400, 4
        X = rng.integers(0, 60, (p, n)).astype(np.float64)
        y = rng.normal(size=n) + X[0] / 30.0
        seed = 50 + case
        F = O.fit(X, y, ntree=1, mtry=p, nodesize=5, seed=seed)
        tr = F.tree(0)
        w = O.bootstrap(seed, 0, n)
        idx = np.repeat(np.arange(n), w)
        m = sk.DecisionTreeRegressor(max_features=None, min_samples_split=6, min_samples_leaf=1, random_state=0)
        m.fit(X.T[idx], y[idx])
        T = m.tree_

        def same(k, j, R):
            # R: distinct in-bag rows of this node.  With continuous y, equal gains mean
            # identical partitions, so a different feature is accepted only if it induces the
            # same partition of R (a true tie: "several results are correct").
            if tr["feature"][k] < 0:
                assert T.children_left[j] == -1
                assert tr["value"][k] == pytest.approx(T.value[j][0][0], rel=1e-12, abs=1e-12)
                return 1
            f, thr = tr["feature"][k], tr["thr"][k]
            L = R[X[f, R] <= thr]
            Rr = np.setdiff1d(R, L)
            jl, jr = T.children_left[j], T.children_right[j]
            if T.feature[j] == f:
                assert T.threshold[j] == thr
            else:
                L2 = R[X[T.feature[j], R] <= T.threshold[j]]
                if not np.array_equal(L, L2):          # same partition with the sides swapped
                    assert np.array_equal(Rr, L2)
                    jl, jr = jr, jl
            return 1 + same(tr["left"][k], jl, L) + same(tr["left"][k] + 1, jr, Rr)

        assert same(0, 0, np.nonzero(w)[0]) == T.node_count == len(tr["feature"])


# ---------------------------------------------------------------- S5 predict
def test_predict_is_tree_average():
    rng = np.random.default_rng(10)
    X, y = rng.normal(size=(4, 120)), rng.normal(size=120)
    F = O.fit(X, y, ntree=7, seed=3)
    Q = rng.normal(size=(4, 50))
    expect = sum(_walk_all(F.tree(i), Q) for i in range(7))
    assert np.allclose(F.predict_sum(Q), expect, rtol=1e-14)


# ---------------------------------------------------------------- S6-S8 importance
def test_finalize_hand_computed():
    d = np.array([[1.0, 0.0], [3.0, 0.0]])
    npur = np.array([[2.0, 4.0], [6.0, 8.0]])
    y = np.array([1.0, 2.0, 3.0])
    r = O.importance_finalize(d, npur, np.array([2.0, 0.0, 6.0]), np.array([1, 0, 2]), y)
    assert r["inc_mse_raw"].tolist() == [2.0, 0.0]
    assert r["inc_mse_sd"][0] == pytest.approx(math.sqrt(0.5), rel=1e-15) and r["inc_mse_sd"][1] == 0.0
    assert r["inc_mse"][0] == pytest.approx(2.0 / math.sqrt(0.5), rel=1e-15) and r["inc_mse"][1] == 0.0
    assert r["inc_node_purity"].tolist() == [4.0, 6.0]
    assert r["oob_mse"] == 0.5
    assert r["rsq"] == pytest.approx(1 - 0.5 / (2.0 / 3.0), rel=1e-15)


def test_importance_identity_perm_zero_unused_zero_signal_first():
    rng = np.random.default_rng(11)
    n, p = 600, 6
    X = rng.normal(size=(p, n))
    X[5] = 1.0                                  # constant column: never used
    y = 3.0 * X[0] + 0.2 * rng.normal(size=n)
    F = O.fit(X, y, ntree=40, seed=4)
    r0 = F.oob_importance(X, y, perm_identity=True)
    assert np.all(r0["d_slots"] == 0.0)
    r = F.oob_importance(X, y)
    assert np.all(r["d_slots"][:, 5] == 0.0) and np.all(r["npur_slots"][:, 5] == 0.0)
    fin = O.importance_finalize(r["d_slots"], r["npur_slots"], r["oob_sum"], r["oob_cnt"], y)
    assert int(np.argmax(fin["inc_mse"])) == 0
    assert int(np.argmax(fin["inc_node_purity"])) == 0
    noise = fin["inc_mse_raw"][1:5]
    assert np.all(np.abs(noise) < 0.05 * fin["inc_mse_raw"][0])
    # OOB rows: T_i empty rows excluded; counts equal number of trees with w = 0
    cnt = np.zeros(n, np.int64)
    for t in range(40):
        cnt += O.bootstrap(4, t, n) == 0
    assert np.array_equal(cnt, r["oob_cnt"])
    assert np.array_equal(r["nout_t"], [(O.bootstrap(4, t, n) == 0).sum() for t in range(40)])


def test_node_purity_invariant_and_oob_vs_heldout():
    from paper_conf_ipps_madougouvln16_b200 import synthetic as S
    Xa, ya = S.gen_mm(n=3000)
    X, y = np.ascontiguousarray(Xa[:, :1500]), ya[:1500]
    Xh, yh = np.ascontiguousarray(Xa[:, 1500:]), ya[1500:]      # held out, same generator
    p, n = X.shape
    T = 30
    F = O.fit(X, y, ntree=T, seed=12, nthreads=4)
    r = F.oob_importance(X, y)
    fin = O.importance_finalize(r["d_slots"], r["npur_slots"], r["oob_sum"], r["oob_cnt"], y)
    # T * sum_m IncNodePurity_m = sum_t (RSS_root,t - sum RSS_leaves,t)  with RSS from the data
    tot = 0.0
    for i in range(T):
        tr = F.tree(i)
        w = O.bootstrap(12, i, n).astype(np.float64)
        leaf = _leaf_index(tr, X)
        inb = w > 0
        mu = np.dot(w, y) / w.sum()
        root = float(np.sum(w * (y - mu) ** 2))
        leaves = 0.0
        for k in np.unique(leaf[inb]):
            s = inb & (leaf == k)
            mk = np.dot(w[s], y[s]) / w[s].sum()
            leaves += float(np.sum(w[s] * (y[s] - mk) ** 2))
        tot += root - leaves
    assert T * fin["inc_node_purity"].sum() == pytest.approx(tot, rel=1e-7)
    # OOB MSE ~ held-out MSE from the same generator (statistical)
    mse_h = np.mean((F.predict_sum(Xh) / T - yh) ** 2)
    assert 0.5 < fin["oob_mse"] / mse_h < 2.0
    assert fin["rsq"] > 0.8


def _leaf_index(tr, X):
    out = np.empty(X.shape[1], np.int64)
    for r in range(X.shape[1]):
        k = 0
        while tr["feature"][k] >= 0:
            k = tr["left"][k] if X[tr["feature"][k], r] <= tr["thr"][k] else tr["left"][k] + 1
        out[r] = k
    return out


def test_tree_range_sharding_is_bit_identical():
    """Global-tree-id keying: trees [2,5) grown alone equal trees 2..4 of the full forest."""
    rng = np.random.default_rng(13)
    X, y = rng.normal(size=(5, 200)), rng.normal(size=200)
    A = O.fit(X, y, ntree=6, seed=21)
    B = O.fit(X, y, ntree=6, seed=21, tree_begin=2, tree_end=5)
    for i in range(3):
        a, b = A.tree(2 + i), B.tree(i)
        for k in a:
            assert np.array_equal(a[k], b[k])


# ---------------------------------------------------------------- S9 PCA
def test_pca_vs_svd_and_trace():
    from oracle.pca import pca
    rng = np.random.default_rng(14)
    n, p = 500, 8
    L = rng.normal(size=(n, 3))
    X = (L @ rng.normal(size=(3, p)) + 0.1 * rng.normal(size=(n, p))).T * np.array([1e6, 1, 1, 1, 1e-3, 1, 1, 1])[:, None]
    r = pca(X, scale=True)
    Z = (X.T - X.T.mean(0)) / X.T.std(0, ddof=1)
    U, s, Vt = np.linalg.svd(Z, full_matrices=False)
    assert np.allclose(r["sdev"], s / math.sqrt(n - 1), rtol=1e-10)
    for j in range(p):
        v = Vt[j] * np.sign(Vt[j][np.argmax(np.abs(Vt[j]))])
        assert np.allclose(r["rotation"][:, j], v, atol=1e-8)
    assert (r["sdev"] ** 2).sum() == pytest.approx(p, rel=1e-12)   # trace of a correlation matrix
    assert np.allclose(r["rotation"].T @ r["rotation"], np.eye(p), atol=1e-12)


def test_pca_planted_axes():
    """Columns with disjoint supports are exactly uncorrelated: the axes are eigenvectors."""
    n = 400
    X = np.zeros((3, n))
    X[0, :100] = np.arange(100) * 3.0
    X[1, 100:250] = np.linspace(-1, 1, 150)
    X[2, 250:] = np.cos(np.arange(150))
    X = X - X.mean(1, keepdims=True)
    # make them exactly orthogonal after centring by Gram-Schmidt
    Q, _ = np.linalg.qr(X.T)
    X = (Q * np.array([5.0, 2.0, 1.0])).T
    from oracle.pca import pca
    r = pca(X, scale=False)
    assert np.allclose(np.abs(r["rotation"]), np.eye(3), atol=1e-10)
    assert np.allclose(r["sdev"] ** 2 * (n - 1), [25.0, 4.0, 1.0], rtol=1e-10)


# ---------------------------------------------------------------- S6-S8 exact-rational pin
@pytest.mark.parametrize("case", range(6))
def test_oob_importance_vs_exact_rational_bruteforce(case):
    """%IncMSE and OOB error of a tiny forest computed in exact rationals
    from brute trees (tests/brute.py: eq.(3) split search, eq.(1) leaf means), with the
    bootstrap multiplicities, mtry draws, node keys and Feistel permutations taken from the
    oracle's RNG as inputs.  n_o differs from n and between trees, so a wrong divisor of
    d_tm = (e_tm - e_t) / n_o (n instead of n_o, or a shared divisor) fails here."""
    from tests.brute import brute_importance
    rng = np.random.default_rng(500 + case)
    n = int(rng.integers(9, 15))
    p = int(rng.integers(2, 4))
    T = 2 if case < 3 else 3
    X = rng.integers(0, 6, (p, n)).astype(np.float64)
    y = rng.integers(-7, 8, n).astype(np.float64)
    seed = 7000 + case
    mtry = p if case % 2 == 0 else max(p - 1, 1)
    F = O.fit(X, y, ntree=T, mtry=mtry, nodesize=1, seed=seed)
    ro = F.oob_importance(X, y)
    cols = [list(c) for c in X]
    trees, ws, perms = [], [], []
    for t in range(T):
        w = O.bootstrap(seed, t, n)
        draw = (lambda k, t=t: O.draw_mtry(seed, t, k, p, mtry)) if mtry < p else None
        ck = lambda k, s, t=t: O.child_key(seed, t, k, s)
        trees.append(brute_tree(cols, list(y), list(w), 1, draw=draw, child_key=ck))
        ws.append(list(w))
        no = int((w == 0).sum())
        perms.append([[O.perm(seed, t, m, no, a) for a in range(no)] for m in range(p)])
    b = brute_importance(cols, list(y), trees, ws, perms)
    assert all(0 < no < n for no in b["nout"])
    assert ro["nout_t"].tolist() == b["nout"]
    scale = max(max(abs(float(v)) for row in b["d"] for v in row), 1e-300)
    for t in range(T):
        assert ro["e_t"][t] == pytest.approx(float(b["e"][t]), rel=1e-12, abs=1e-12)
        for m in range(p):
            assert abs(ro["d_slots"][t, m] - float(b["d"][t][m])) <= 1e-12 * scale, (t, m)
    assert ro["oob_cnt"].tolist() == b["ocnt"]
    assert np.allclose(ro["oob_sum"], [float(v) for v in b["osum"]], rtol=1e-13, atol=1e-12)
    fin = O.importance_finalize(ro["d_slots"], ro["npur_slots"], ro["oob_sum"], ro["oob_cnt"], y)
    for m in range(p):
        assert fin["inc_mse_raw"][m] == pytest.approx(float(b["raw"][m]), rel=1e-12, abs=1e-12 * scale)
        assert fin["inc_mse_sd"][m] == pytest.approx(b["sd"][m], rel=1e-9, abs=1e-12 * scale)
        if b["sd"][m] >= np.finfo(float).eps:
            assert fin["inc_mse"][m] == pytest.approx(float(b["raw"][m]) / b["sd"][m], rel=1e-9)
    assert fin["oob_mse"] == pytest.approx(float(b["oob_mse"]), rel=1e-13)
    assert fin["rsq"] == pytest.approx(float(b["rsq"]), rel=1e-12, abs=1e-13)


def test_oob_importance_exact_pin_is_not_vacuous():
    """At least one of the pinned tiny forests has a nonzero d_tm in every tree with n_o > 0,
    so the exact pin above tests the divisor rather than comparing zeros."""
    from tests.brute import brute_importance
    hits = 0
    for case in range(6):
        rng = np.random.default_rng(500 + case)
        n = int(rng.integers(9, 15))
        p = int(rng.integers(2, 4))
        T = 2 if case < 3 else 3
        X = rng.integers(0, 6, (p, n)).astype(np.float64)
        y = rng.integers(-7, 8, n).astype(np.float64)
        seed = 7000 + case
        mtry = p if case % 2 == 0 else max(p - 1, 1)
        F = O.fit(X, y, ntree=T, mtry=mtry, nodesize=1, seed=seed)
        ro = F.oob_importance(X, y)
        if all(np.any(ro["d_slots"][t] != 0.0) for t in range(T)):
            hits += 1
    assert hits >= 3
