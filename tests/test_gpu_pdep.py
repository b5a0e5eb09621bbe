"""GPU parity of partial dependence (bf_pd_grid, bf_partial_dependence)
against oracle/pdep.py.  Bar: grid bit-exact (same fp64 operations);
pd_sum / pd within 1e-9 relative (sums of fp64 leaf values in another order,
DESIGN.md R22)."""
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
from oracle import pdep as PD  # noqa: E402

DEV = torch.device("cuda:0")


def dev(a):
    return torch.from_numpy(np.ascontiguousarray(a)).to(DEV)


def test_grid_bit_exact():
    rng = np.random.default_rng(1)
    cols = [rng.normal(size=1000), np.round(rng.normal(size=777) * 3), np.full(50, 2.5),
            np.array([-0.0, 0.0, 1.0, 1.0]), rng.integers(0, 5, 333).astype(np.float64), np.arange(5000.0) * 1e-3]
    for x in cols:
        for n_pt in (1, 7, 51):
            g = bf.pd_grid(dev(x), n_pt).cpu().numpy()
            o = PD.pd_grid(x, n_pt)
            assert g.tobytes() == o.tobytes(), (x[:5], n_pt)
    g = bf.pd_grid(np.ascontiguousarray(cols[0]), 51)  # host pointer path
    assert g.tobytes() == PD.pd_grid(cols[0], 51).tobytes()


@pytest.mark.parametrize("cfg,T,n_rows", [("C1", 40, None), ("C2", 12, 1000)])
def test_partial_dependence_matches_oracle(cfg, T, n_rows):
    X, y, _ = S.dataset(cfg)
    seed = S.FOREST_SEED + 7
    gf = bf.fit(dev(X), dev(y), ntree=T, seed=seed)
    of = O.fit(X, y, ntree=T, seed=seed, nthreads=4)
    Xa = X if n_rows is None else np.ascontiguousarray(X[:, :n_rows])  # ragged row count
    p = X.shape[0]
    for m in (0, p // 2, p - 1):
        grid, ps, pd = gf.partial_dependence(dev(Xa), m)
        og = PD.pd_grid(Xa[m], 51)
        assert grid.cpu().numpy().tobytes() == og.tobytes()
        os_, opd = PD.partial_dependence(of, Xa, m, og)
        assert np.allclose(ps.cpu().numpy(), os_, rtol=1e-9, atol=0)
        assert np.allclose(pd.cpu().numpy(), opd, rtol=1e-9, atol=0)


def test_partial_dependence_single_point_host_path_and_shards():
    X, y, _ = S.dataset("C1")
    seed = S.FOREST_SEED + 3
    T = 16
    of = O.fit(X, y, ntree=T, seed=seed, nthreads=4)
    grid = np.array([float(np.median(X[2]))])
    os_, opd = PD.partial_dependence(of, X, 2, grid)
    # host arrays through the C ABI
    gf = bf.fit(dev(X), dev(y), ntree=T, seed=seed)
    _, ps, pd = gf.partial_dependence(np.ascontiguousarray(X), 2, grid=grid)
    assert np.allclose(ps, os_, rtol=1e-9, atol=0) and np.allclose(pd, opd, rtol=1e-9, atol=0)
    # tree shards: pd_sum of disjoint ranges add up (the multi-GPU all-reduce)
    a = bf.fit(dev(X), dev(y), ntree=T, seed=seed, tree_begin=0, tree_end=5)
    b = bf.fit(dev(X), dev(y), ntree=T, seed=seed, tree_begin=5, tree_end=T)
    _, sa, _ = a.partial_dependence(dev(X), 2, grid=dev(grid), ntree_total=T)
    _, sb, _ = b.partial_dependence(dev(X), 2, grid=dev(grid), ntree_total=T)
    assert np.allclose((sa + sb).cpu().numpy(), os_, rtol=1e-9, atol=0)
