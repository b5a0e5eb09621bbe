"""GPU parity of the varimax rotation (bf_varimax) against oracle/varimax.py.
Bar: same iteration count; loadings and rotation within 1e-9 (absolute, the
entries are O(1)): both sides take the polar factor U V^T of the same B, whose
value does not depend on the SVD algorithm (LAPACK vs one-sided Jacobi)."""
from __future__ import annotations

import numpy as np
import pytest

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():
    pytest.skip("no CUDA device", allow_module_level=True)

import paper_conf_ipps_madougouvln16_b200 as bf  # noqa: E402
from paper_conf_ipps_madougouvln16_b200 import synthetic as S  # noqa: E402
from oracle import pca as OP  # noqa: E402
from oracle import varimax as V  # noqa: E402

DEV = torch.device("cuda:0")


def _gpu(L, normalize=True, eps=1e-5, host=False):
    Lc = np.ascontiguousarray(L.T)  # (k, p) = column-major p x k
    arg = Lc if host else torch.from_numpy(Lc).to(DEV)
    r = bf.varimax(arg, normalize=normalize, eps=eps)
    lo = r["loadings"] if host else r["loadings"].cpu().numpy()
    ro = r["rotmat"] if host else r["rotmat"].cpu().numpy()
    return lo.T, ro.T, r["iters"]


def test_varimax_on_counter_pca_loadings():
    X, y, _ = S.dataset("C3")
    pc = OP.pca(X, scale=True)
    for k in (2, 4, 8):
        L = V.loadings_from_pca(pc["rotation"], pc["sdev"], k)
        z, T, it = V.varimax(L)
        gz, gT, git = _gpu(L)
        assert git == it
        assert np.allclose(gz, z, atol=1e-9, rtol=0) and np.allclose(gT, T, atol=1e-9, rtol=0)


@pytest.mark.parametrize("p,k,normalize,eps", [(64, 10, True, 1e-5), (20, 2, False, 1e-12), (33, 5, True, 1e-9),
                                               (7, 7, True, 1e-5)])
def test_varimax_random(p, k, normalize, eps):
    rng = np.random.default_rng(p * 100 + k)
    L = rng.normal(size=(p, k))
    z, T, it = V.varimax(L, normalize=normalize, eps=eps)
    gz, gT, git = _gpu(L, normalize, eps)
    assert git == it
    assert np.allclose(gz, z, atol=1e-9, rtol=0) and np.allclose(gT, T, atol=1e-9, rtol=0)


def test_varimax_single_factor_and_host_path():
    L = np.arange(1.0, 7.0).reshape(6, 1)
    gz, gT, git = _gpu(L, host=True)
    assert git == 0 and np.array_equal(gz, L) and gT.tolist() == [[1.0]]
    rng = np.random.default_rng(3)
    L = rng.normal(size=(15, 3))
    z, T, it = V.varimax(L)
    gz, gT, git = _gpu(L, host=True)
    assert git == it and np.allclose(gz, z, atol=1e-9, rtol=0)
