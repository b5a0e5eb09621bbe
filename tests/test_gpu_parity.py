"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle.

Bar (BASELINE north_star): bootstrap/OOB indices and tree topology
(feature, threshold, structure, counts) bit-exact; node values and
predictions within 1e-9 relative; OOB MSE and %IncMSE within 1e-6
relative; importance ranking identical.
"""
from __future__ import annotations

import math
import os
import random

import numpy as np
import pytest

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():
    pytest.skip("no CUDA device", allow_module_level=True)

import paper_conf_ipps_madougouvln16_b200 as bf  # noqa: E402
from paper_conf_ipps_madougouvln16_b200 import synthetic as S  # noqa: E402
from oracle import oracle as O  # noqa: E402
from tests.helpers import assert_same_ranking, compare_forest, eigen_clusters, rel_close  # noqa: E402

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")
DEV = torch.device("cuda:0")


def dev(a):
    return torch.from_numpy(np.ascontiguousarray(a)).to(DEV)


# ------------------------------------------------------------------ primitives
def test_philox_kat_and_random_counters():
    rows = [l.split() for l in open(os.path.join(GOLDEN, "philox_kat.txt")) if l.strip() and not l.startswith("#")]
    for r in rows:
        v = [int(x, 16) for x in r]
        out = bf.philox(np.array([v[0:4]], np.uint32), v[4], v[5])
        assert out[0].tolist() == v[6:10]
    rng = np.random.default_rng(0)
    ctr = rng.integers(0, 2 ** 32, (1000, 4), dtype=np.uint64).astype(np.uint32)
    out = bf.philox(ctr, 0xDEADBEEF, 0x12345678)
    for i in range(0, 1000, 97):
        assert out[i].tolist() == O.philox(ctr[i].tolist(), [0xDEADBEEF, 0x12345678])


def test_int128_to_double_correct_rounding():
    rng = random.Random(5)
    vals = [0, 1, -1, (1 << 53) + 1, ((1 << 53) + 1) << 40, (1 << 127) - 1, -(1 << 127), ((1 << 54) + 3) << 30]
    for _ in range(20000):
        b = rng.randrange(1, 127)
        v = rng.getrandbits(b)
        if rng.random() < 0.4:
            v = (((rng.getrandbits(53) | (1 << 53)) * 2 + 1) << rng.randrange(0, 60)) & ((1 << 126) - 1)
            if rng.random() < 0.5:
                v += rng.choice([-1, 1])
        vals.append(-v if rng.random() < 0.5 else v)
    hi = np.array([(v >> 64) for v in vals], dtype=object)
    hi = np.array([int(h) for h in hi], np.int64)
    lo = np.array([v & ((1 << 64) - 1) for v in vals], dtype=np.uint64)
    got = bf.i128_to_double(hi, lo)
    exp = np.array([float(v) for v in vals])
    assert np.array_equal(got, exp)


@pytest.mark.parametrize("n", [1, 2, 7, 256, 4096, 100003])
def test_fixed_point_bit_exact(n):
    rng = np.random.default_rng(n)
    y = rng.lognormal(0, 2, n) * rng.choice([-1, 1], n)
    yq_o, q_o = O.fixed_point(y)
    yq_g, q_g = bf.fixed_point(dev(y))
    assert q_g == q_o
    assert np.array_equal(yq_g.cpu().numpy(), yq_o)


@pytest.mark.parametrize("n", [1, 3, 256, 4096, 1_000_000])
def test_bootstrap_bit_exact(n):
    seed = 0xBF10_0004
    w = bf.bootstrap(seed, 5, 3, n)
    for k in range(3):
        assert np.array_equal(w[k], O.bootstrap(seed, 5 + k, n))


@pytest.mark.parametrize("n_o", [1, 2, 3, 5, 17, 1000, 4097, 65536])
def test_feistel_perm_bit_exact(n_o):
    g = bf.perm(77, 3, 11, n_o)
    assert sorted(g.tolist()) == list(range(n_o))
    idx = range(n_o) if n_o <= 5000 else range(0, n_o, 61)
    for a in idx:
        assert g[a] == O.perm(77, 3, 11, n_o, a)


# ------------------------------------------------------------------ fit topology
CASES = [
    # (n, p, kind, ntree, mtry, nodesize, small_node_max, trees_in_flight)
    (40, 3, "int", 6, 0, 1, 0, 0),
    (40, 3, "int", 6, 3, 1, 2, 0),          # global phase only (A = 2)
    (300, 5, "mixed", 8, 0, 5, 8, 3),       # deep global phase, ragged batches
    (300, 5, "mixed", 8, 0, 5, 0, 0),       # subtree kernel only
    (1000, 7, "cont", 5, 7, 1, 64, 2),      # mtry = p, nodesize 1
    (2500, 12, "int", 4, 0, 5, 300, 0),
    (777, 1, "cont", 3, 1, 2, 16, 0),       # p = 1
    (5, 2, "int", 3, 0, 5, 0, 0),           # root is a leaf (n <= nodesize)
    (6, 2, "int", 3, 0, 1, 0, 0),
]


@pytest.mark.parametrize("case", CASES)
def test_fit_topology_bit_exact(case):
    n, p, kind, T, mtry, ns, A, B = case
    X, y = S.small_random(n, p, seed=n * 31 + p, kind=kind)
    seed = 1234 + n
    of = O.fit(X, y, ntree=T, mtry=mtry, nodesize=ns, seed=seed, nthreads=4)
    gf = bf.fit(dev(X), dev(y), ntree=T, mtry=mtry, nodesize=ns, seed=seed, small_node_max=A, trees_in_flight=B)
    assert compare_forest(gf, of) > 0
    assert gf.info.q == of.q


def test_fit_degenerate_inputs():
    rng = np.random.default_rng(1)
    X = rng.normal(size=(3, 50))
    # constant y -> single leaves
    gf = bf.fit(dev(X), dev(np.full(50, 2.5)), ntree=3, seed=1)
    e = gf.export()
    assert np.all(e["feature"] == -1) and np.all(e["thr_or_value"] == 2.5)
    # constant X -> single leaves
    y = rng.normal(size=50)
    of = O.fit(np.ones((3, 50)), y, ntree=3, seed=2)
    gf = bf.fit(dev(np.ones((3, 50))), dev(y), ntree=3, seed=2)
    compare_forest(gf, of)
    # -0.0 / +0.0 are one value
    X2 = np.zeros((2, 60))
    X2[0, ::2] = -0.0
    X2[1] = rng.integers(0, 3, 60)
    y2 = np.concatenate([y, y[:10]])
    of = O.fit(X2, y2, ntree=4, seed=3, nodesize=1)
    gf = bf.fit(dev(X2), dev(y2), ntree=4, seed=3, nodesize=1)
    compare_forest(gf, of)
    # NaN rejected
    Xn = X.copy()
    Xn[1, 7] = np.nan
    with pytest.raises(bf.BFError) as ei:
        bf.fit(dev(Xn), dev(y), ntree=1)
    assert ei.value.code == -2


def test_fit_host_pointers_equal_device_pointers():
    X, y = S.small_random(500, 6, seed=9)
    of = O.fit(X, y, ntree=4, seed=5, nthreads=4)
    a = bf.fit(dev(X), dev(y), ntree=4, seed=5)
    b = bf.fit(X, y, ntree=4, seed=5)            # host numpy: staged by the library
    assert compare_forest(a, of) > 0
    assert compare_forest(b, of) > 0             # the host-pointer forest walked against the oracle
    Q = S.gen_query(X, 777)
    ys_h, _ = b.predict(Q, ntree_total=4)        # host query, host outputs
    assert rel_close(ys_h, of.predict_sum(Q), 1e-9)


def test_tree_range_sharding_bit_identical():
    X, y = S.gen_reduction()
    full = O.fit(X, y, ntree=10, seed=77)
    part = bf.fit(dev(X), dev(y), ntree=10, seed=77, tree_begin=3, tree_end=7)
    e = part.export()
    from tests.helpers import compare_tree
    for i in range(4):
        lo, hi = e["tree_off"][i], e["tree_off"][i + 1]
        g = {k: e[k][lo:hi] for k in ("feature", "left", "thr_or_value", "count", "value", "drss")}
        compare_tree(g, full.tree(3 + i))


# ------------------------------------------------------------------ configs C1..C3 in full
def _config_data(cfg):
    X, y, c = S.dataset(cfg)
    if cfg == "C3":
        from oracle.pca import pca, n_components
        r = pca(X, scale=True)
        k = n_components(r["sdev"])
        X = np.ascontiguousarray(np.concatenate([r["scores"][:, :k].T, c.extra["L"][None, :], c.extra["M"]], axis=0))
    return X, y, c


@pytest.mark.parametrize("cfg", ["C1", "C2", "C3"])
def test_config_forest_parity(cfg):
    X, y, c = _config_data(cfg)
    T = c.ntree if cfg == "C1" else 60
    of = O.fit(X, y, ntree=T, seed=S.FOREST_SEED + 1, nthreads=os.cpu_count() or 4)
    gf = bf.fit(dev(X), dev(y), ntree=T, seed=S.FOREST_SEED + 1)
    compare_forest(gf, of)
    # predictions
    Q = S.gen_query(X, 5000)
    ys, yh = gf.predict(dev(Q), ntree_total=T)
    po = of.predict_sum(Q)
    assert rel_close(ys.cpu().numpy(), po, 1e-9)
    assert rel_close(yh.cpu().numpy(), po / T, 1e-9)


# ------------------------------------------------------------------ OOB importance
@pytest.mark.parametrize("cfg", ["C1", "C2"])
def test_oob_importance_parity(cfg):
    X, y, c = _config_data(cfg)
    T = 120 if cfg == "C1" else 40
    seed = S.FOREST_SEED + 2
    of = O.fit(X, y, ntree=T, seed=seed, nthreads=os.cpu_count() or 4)
    ro = of.oob_importance(X, y)
    gf = bf.fit(dev(X), dev(y), ntree=T, seed=seed)
    rg = gf.oob_importance(dev(X), dev(y))
    rg = {k: v.cpu().numpy() for k, v in rg.items()}
    assert np.array_equal(rg["nout_t"], ro["nout_t"])
    assert np.array_equal(rg["oob_cnt"], ro["oob_cnt"])
    assert rel_close(rg["oob_sum"], ro["oob_sum"], 1e-9)
    assert rel_close(rg["e_t"], ro["e_t"], 1e-9)
    # d_tm: exact zeros where the oracle has exact zeros (unused predictors)
    unused = ro["npur_slots"] == 0.0
    assert np.all(rg["d_slots"][unused] == 0.0)
    assert rel_close(rg["d_slots"], ro["d_slots"], 1e-6, 1e-9)
    assert rel_close(rg["npur_slots"], ro["npur_slots"], 1e-9, 1e-12)
    fo = O.importance_finalize(ro["d_slots"], ro["npur_slots"], ro["oob_sum"], ro["oob_cnt"], y)
    fg = bf.importance_finalize(dev(rg["d_slots"]), dev(rg["npur_slots"]), dev(rg["oob_sum"]), dev(rg["oob_cnt"]), dev(y))
    fg = {k: (v.cpu().numpy() if hasattr(v, "cpu") else v) for k, v in fg.items()}
    assert rel_close(fg["inc_mse_raw"], fo["inc_mse_raw"], 1e-6, 1e-9)
    assert rel_close(fg["inc_mse"], fo["inc_mse"], 1e-6, 1e-9)
    assert rel_close(fg["inc_node_purity"], fo["inc_node_purity"], 1e-9)
    assert abs(float(fg["oob_mse"]) - fo["oob_mse"]) <= 1e-6 * fo["oob_mse"]
    assert abs(float(fg["rsq"]) - fo["rsq"]) <= 1e-6 * abs(fo["rsq"]) + 1e-12
    # ranking identical: a pair may be ordered differently only if its own two values tie within 1e-12
    assert_same_ranking(fg["inc_mse"], fo["inc_mse"], 1e-12, tag=f"{cfg} %IncMSE")
    assert_same_ranking(fg["inc_node_purity"], fo["inc_node_purity"], 1e-12, tag=f"{cfg} IncNodePurity")


# ------------------------------------------------------------------ PCA
@pytest.mark.parametrize("scale", [True, False])
def test_pca_parity(scale):
    from oracle.pca import pca
    X, _, _ = S.dataset("C3") if scale else (S.gen_mm(2048)[0], None, None)
    ro = pca(X, scale=scale)
    k = 6
    rg = bf.pca(dev(X), scale=scale, k=k)
    sd = rg["sdev"].cpu().numpy()
    # backward-stable eigensolvers: |lambda_gpu - lambda_oracle| <= c * eps * lambda_max (Weyl)
    lam_g, lam_o = sd ** 2, ro["sdev"] ** 2
    assert np.all(np.abs(lam_g - lam_o) <= 1e-9 * lam_o + 1e-12 * lam_o[0])
    rot = rg["rotation"].cpu().numpy()  # row j = component j
    V = ro["rotation"]                  # column j = component j
    lam = ro["sdev"] ** 2
    # eigenvectors of a well-separated eigenvalue: unique up to the sign rule, compared directly;
    # a degenerate cluster (gap <= 1e-6 lambda_0): compared by its projector (reading R16)
    for grp in eigen_clusters(lam, 1e-6):
        Pg = rot[grp].T @ rot[grp]
        Po = V[:, grp] @ V[:, grp].T
        assert np.allclose(Pg, Po, atol=1e-7), f"projector of components {grp}"
        if len(grp) == 1:
            assert np.allclose(rot[grp[0]], V[:, grp[0]], atol=1e-7)
    # scores: equal to Z V_k by definition (S9); per component where unique, by projector otherwise
    mu = X.mean(axis=1)
    Z = (X - mu[:, None]).T
    if scale:
        Z = Z / X.std(axis=1, ddof=1)
    sc = rg["scores"].cpu().numpy()     # row j = scores of component j
    so = ro["scores"]                   # column j
    for grp in eigen_clusters(lam, 1e-6):
        g_in = [j for j in grp if j < k]
        if not g_in:
            continue
        atol = 1e-7 * np.abs(so).max()
        assert np.allclose(sc[g_in].T, Z @ rot[g_in].T, rtol=1e-7, atol=atol), f"scores {g_in} != Z V"
        if len(g_in) == len(grp):       # whole cluster retained: its score projection is basis-free
            assert np.allclose(sc[g_in].T @ rot[g_in], so[:, g_in] @ V[:, g_in].T, rtol=1e-7, atol=atol)
        if len(grp) == 1:
            assert np.allclose(sc[grp[0]], so[:, grp[0]], rtol=1e-7, atol=atol)


def test_pca_retained_parity():
    """Retained components (reading R15) on the device vs the oracle's cumulative-share rule, on real
    PCA spectra, on spectra where the share crosses 0.97 exactly at a component, and at the cap."""
    from oracle.pca import n_components, pca
    cases = [pca(S.dataset("C3")[0], scale=True)["sdev"], pca(S.gen_mm(2048)[0], scale=True)["sdev"],
             np.sqrt(np.array([97.0, 2.0, 1.0])), np.sqrt(np.array([96.0, 1.0, 1.0, 1.0, 1.0])),
             np.ones(30), np.sqrt(np.linspace(30, 1, 30)), np.array([1.0])]
    for sd in cases:
        for cap in (1, 3, 10):
            assert bf.pca_retained(dev(sd), 0.97, cap) == n_components(sd, 0.97, cap), (sd, cap)
            assert bf.pca_retained(np.ascontiguousarray(sd), 0.97, cap) == n_components(sd, 0.97, cap)


# ------------------------------------------------------------------ C4 at full size, sampled trees
@pytest.mark.slow
def test_c4_full_size_sampled_trees():
    X, y = S.gen_scaled()
    seed = S.FOREST_SEED + 4
    trees = (0, 1)
    of = O.fit(X, y, ntree=1000, seed=seed, tree_begin=0, tree_end=2, nthreads=2)
    gf = bf.fit(dev(X), dev(y), ntree=1000, seed=seed, tree_begin=0, tree_end=2)
    compare_forest(gf, of)
    Q = S.gen_query(X, 2000)
    ys, _ = gf.predict(dev(Q))
    assert rel_close(ys.cpu().numpy(), of.predict_sum(Q), 1e-9)


# ------------------------------------------------------------------ C4 in the bench.py launch configuration
def test_c4_bench_configuration_sampled():
    """The whole 1000-tree C4 forest fitted as bench.py fits it (batches of trees in flight), sampled trees
    from the first, a middle and the last batch compared with the oracle bit for bit; predictions of the
    10M-row query batch (generated on the device as bench.py does) checked on sampled rows against a host
    walk of the exported forest; importance slots of the sampled trees against the oracle's."""
    from concurrent.futures import ThreadPoolExecutor
    from tests.helpers import compare_tree
    X, y = S.gen_scaled()
    p, n = X.shape
    T, seed = 1000, S.FOREST_SEED + 4
    Xd, yd = dev(X), dev(y)
    gf = bf.fit(Xd, yd, ntree=T, seed=seed)
    sample = (0, 136, 517, 731, 999)  # trees of 5 different batches (37 trees in flight)
    with ThreadPoolExecutor(len(sample)) as ex:  # ctypes releases the GIL: one oracle tree per host thread
        ofs = list(ex.map(lambda t: O.fit(X, y, ntree=T, seed=seed, tree_begin=t, tree_end=t + 1), sample))
    e = gf.export()
    for t, of in zip(sample, ofs):
        lo, hi = e["tree_off"][t], e["tree_off"][t + 1]
        compare_tree({k: e[k][lo:hi] for k in ("feature", "left", "thr_or_value", "count", "value", "drss")},
                     of.tree(0), tag=f"tree {t}")
    # 10M query rows drawn on the device exactly as bench.py draws them
    m = 10_000_000
    g = torch.Generator(device=DEV)
    g.manual_seed(S.QUERY_SEED)
    idx = torch.randint(0, n, (m,), device=DEV, generator=g)
    Qd = Xd[:, idx]
    jit = torch.rand((p, m), device=DEV, generator=g) < 0.5
    Qd = torch.where(jit, Qd * (1.0 + 0.01 * torch.randn((p, m), device=DEV, generator=g, dtype=torch.float64)), Qd)
    Qd = Qd.contiguous()
    del idx, jit
    ys, _ = gf.predict(Qd, ntree_total=T)
    rows = np.random.default_rng(3).integers(0, m, 48)
    Qs = Qd[:, torch.from_numpy(rows).to(DEV)].cpu().numpy()
    got = ys[torch.from_numpy(rows).to(DEV)].cpu().numpy()
    del Qd, ys
    feat, left, thr, off = e["feature"], e["left"], e["thr_or_value"], e["tree_off"]
    ref = np.zeros(len(rows))
    for t in range(T):
        base = off[t]
        for r in range(len(rows)):
            k = 0
            while feat[base + k] >= 0:
                k = left[base + k] + (0 if Qs[feat[base + k], r] <= thr[base + k] else 1)
            ref[r] += thr[base + k]
    assert rel_close(got, ref, 1e-9)
    # the sampled trees alone (bf_forest_import of their exported arrays), predicted on the device over the
    # sampled query rows, against the oracle's trees (S5): the GPU prediction path checked by the oracle itself
    trees = [{k: e[k][e["tree_off"][t]:e["tree_off"][t + 1]] for k in ("feature", "left", "thr_or_value", "count",
                                                                       "value", "drss")} for t in sample]
    arrays = {k: np.concatenate([tr[k] for tr in trees]) for k in trees[0]}
    arrays["tree_off"] = np.concatenate([[0], np.cumsum([tr["feature"].size for tr in trees])]).astype(np.int64)
    info = e["info"]
    info.tree_begin, info.tree_end, info.ntree_total = 0, len(sample), len(sample)
    info.total_nodes = int(arrays["tree_off"][-1])
    sub = bf.forest_import(arrays, info)
    ys_sub, _ = sub.predict(dev(Qs), ntree_total=len(sample))
    ref_sub = sum(of.predict_sum(Qs) for of in ofs)
    assert rel_close(ys_sub.cpu().numpy(), ref_sub, 1e-9)
    sub.free()
    # importance slots of the sampled trees (S7) in the batched launch configuration
    acc = gf.oob_importance(Xd, yd)
    d = acc["d_slots"].cpu().numpy()
    npu = acc["npur_slots"].cpu().numpy()
    ros = [of.oob_importance(X, y) for of in ofs]
    for t, ro in zip(sample, ros):
        assert int(acc["nout_t"][t]) == int(ro["nout_t"][0])
        assert rel_close(d[t], ro["d_slots"][0], 1e-6, atol_scale=1e-9)
        assert rel_close(npu[t], ro["npur_slots"][0], 1e-9, atol_scale=1e-12)
        assert np.all(d[t][ro["npur_slots"][0] == 0.0] == 0.0)   # predictors unused by tree t: exactly 0
    # finalize (S7/S8 aggregation) over the sampled trees' slots, GPU kernel vs oracle, and the ranking
    do = np.stack([ro["d_slots"][0] for ro in ros])
    no = np.stack([ro["npur_slots"][0] for ro in ros])
    osum = sum(ro["oob_sum"] for ro in ros)
    ocnt = sum(ro["oob_cnt"] for ro in ros).astype(np.int32)
    fo = O.importance_finalize(do, no, osum, ocnt, y)
    fg = bf.importance_finalize(dev(d[list(sample)]), dev(npu[list(sample)]), dev(osum), dev(ocnt), yd)
    fg = {k: (v.cpu().numpy() if hasattr(v, "cpu") else v) for k, v in fg.items()}
    assert rel_close(fg["inc_mse_raw"], fo["inc_mse_raw"], 1e-6, 1e-9)
    assert rel_close(fg["inc_mse"], fo["inc_mse"], 1e-6, 1e-9)
    assert rel_close(fg["inc_node_purity"], fo["inc_node_purity"], 1e-9, 1e-12)
    assert_same_ranking(fg["inc_mse"], fo["inc_mse"], 1e-12, tag="C4 sampled %IncMSE")
    assert_same_ranking(fg["inc_node_purity"], fo["inc_node_purity"], 1e-12, tag="C4 sampled IncNodePurity")


_TQ_SCRIPT = r"""
import sys
sys.path.insert(0, sys.argv[1])
import torch
import paper_conf_ipps_madougouvln16_b200 as bf
from paper_conf_ipps_madougouvln16_b200 import synthetic as S
from oracle import oracle as O
from tests.helpers import compare_forest
X, y = S.small_random(2500, 12, seed=4242, kind="mixed")
of = O.fit(X, y, ntree=8, nodesize=1, seed=99, nthreads=4)
gf = bf.fit(torch.from_numpy(X).cuda(), torch.from_numpy(y).cuda(), ntree=8, nodesize=1, seed=99, small_node_max=0)
assert compare_forest(gf, of) > 0
print("ok")
"""


@pytest.mark.parametrize("env", [{"BF_TQ_BIGGER_FIRST": "0"}, {"BF_TQ_BIGGER_FIRST": "1", "BF_TQ_SLEEP_MAX": "32"},
                                 {"BF_SUBTREE_PACK": "0"}, {"BF_TINY_V": "0"}, {"BF_TINY_V": "1", "BF_TINY_MAX": "128"},
                                 {"BF_TQ_LPT": "0"}, {"BF_TINY_V": "1"}, {"BF_TINY_V": "2"}, {"BF_TINY_MAX": "128"},
                                 {"BF_SUBTREE_HW": "4"}, {"BF_SUBTREE_HW": "2"}])
def test_tiny_queue_schedule_does_not_change_the_forest(env):
    """The subtree kernel's tiny-node queue order (which child keeps the warp, idle back-off) and the packing of
    several small roots (of different trees) into one CTA are scheduling only:
    every node's split depends on its own rows and Philox key, so the forest stays bit-exact vs the oracle.
    So are the tiny-node search variants (BF_TINY_V=0: staged warp items over tiny roots of <= 64 rows;
    BF_TINY_V=1: lane per drawn feature with a position table built for all tiny roots at the phase start, also
    over tiny roots of up to 128 rows; BF_TINY_V=2: ballot-built member masks; the default BF_TINY_V=3: the
    position table built per tiny root by the warp that takes it) and the helper warps that grow tiny nodes while
    the others run the medium levels (BF_SUBTREE_HW=2 / 4, with the ballot masks).
    The switches are read once per process, hence the subprocess."""
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    r = subprocess.run([sys.executable, "-c", _TQ_SCRIPT, root], env={**os.environ, **env}, cwd=root,
                       capture_output=True, text=True, timeout=600)
    assert r.returncode == 0 and r.stdout.strip().endswith("ok"), r.stderr[-2000:]


def test_empty_tree_range_is_an_empty_forest():
    """ntree < ranks gives some rank an empty range [b, b): honoured as an empty forest (not the whole
    forest), and predict / importance of it contribute exact zeros to the all-reduces."""
    X, y = S.small_random(200, 4, seed=3)
    Xd, yd = dev(X), dev(y)
    e = bf.fit(Xd, yd, ntree=3, seed=8, tree_begin=0, tree_end=0)
    assert e.info.tree_end - e.info.tree_begin == 0 and e.info.total_nodes == 0
    ys, _ = e.predict(Xd, ntree_total=3)
    assert torch.all(ys == 0)
    acc = e.oob_importance(Xd, yd)
    assert acc["d_slots"].numel() == 0 and torch.all(acc["oob_cnt"] == 0) and torch.all(acc["oob_sum"] == 0)
    w = bf.fit(Xd, yd, ntree=3, seed=8, tree_begin=3, tree_end=3)
    assert w.info.total_nodes == 0
    full = bf.fit(Xd, yd, ntree=3, seed=8)
    assert full.info.tree_end - full.info.tree_begin == 3


def test_library_memory_comes_from_the_torch_caching_allocator():
    """bf_set_allocator is installed with torch's caching allocator by the binding: a forest's device arrays are
    torch allocations (memory_allocated grows while it lives and drops when it is freed), and the fit's work
    space is returned to torch's pool (reserved, not allocated) after bf_fit, except the node-list work space the
    library keeps across fits (sized by the first fit of a shape, reused by the next: a warm-up fit precedes the
    measurement, and the measured fit allocates no more list space)."""
    assert bf.torch_allocator_active()
    X, y = S.small_random(3000, 8, seed=21)
    Xd, yd = dev(X), dev(y)
    bf.fit(Xd, yd, ntree=8, seed=3).free()  # sizes the held list work space for this shape
    torch.cuda.synchronize()
    a0 = torch.cuda.memory_allocated()
    f = bf.fit(Xd, yd, ntree=8, seed=3)
    torch.cuda.synchronize()
    a1 = torch.cuda.memory_allocated()
    nodes = f.info.total_nodes
    assert a1 - a0 >= nodes * 16          # at least the 16-byte node array
    ys, _ = f.predict(Xd, ntree_total=8)  # the lazily built compact copy also comes from torch
    side = torch.cuda.Stream()
    with torch.cuda.stream(side):         # a call on another stream: free waits for the device
        ys2, _ = f.predict(Xd, ntree_total=8)
    f.free()
    torch.cuda.synchronize()
    assert torch.cuda.memory_allocated() - a0 <= 2 * ys.numel() * 8 * 2 + 4096
    assert torch.equal(ys, ys2)
    del ys, ys2
    a2 = torch.cuda.memory_allocated()
    bf.release_workspace()                # the held list buffers go back to torch's pool
    torch.cuda.synchronize()
    assert torch.cuda.memory_allocated() < a2
