"""GPU tests of the hand-written device primitives (csrc/prims.cu) under the presort (SURVEY 8(a) row a3,
P:81-91) and the per-level offsets of the fit: the LSD radix sort against numpy's stable argsort (keys with
heavy ties, several segments, ragged tile tails, digits constant in every key), the prefix scans against
numpy cumsum, unique against numpy.unique.  Integer work: bit-exact."""
from __future__ import annotations

import numpy as np
import pytest

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():
    pytest.skip("no CUDA device", allow_module_level=True)

import paper_conf_ipps_madougouvln16_b200 as bf  # noqa: E402

DEV = torch.device("cuda:0")


def _keys(rng, n, kind):
    if kind == "full":
        return rng.integers(0, 2 ** 63, n, dtype=np.uint64) * np.uint64(2) + rng.integers(0, 2, n, dtype=np.uint64)
    if kind == "ties":
        return rng.integers(0, 37, n).astype(np.uint64) << np.uint64(40)
    if kind == "doubles":  # order-preserving keys of lognormal counts (the presort's keys)
        x = np.floor(rng.lognormal(3, 2, n))
        b = x.view(np.uint64)
        return np.where(b >> np.uint64(63), ~b, b | np.uint64(1 << 63))
    raise KeyError(kind)


@pytest.mark.parametrize("n,nseg,kind", [(1, 1, "full"), (2, 1, "ties"), (4095, 1, "full"), (4097, 3, "ties"),
                                         (100_003, 1, "doubles"), (65_536, 5, "doubles"), (1_000_003, 2, "full")])
def test_radix_sort_pairs_stable(n, nseg, kind):
    rng = np.random.default_rng(n + nseg)
    k = _keys(rng, n * nseg, kind)
    v = np.tile(np.arange(n, dtype=np.uint32), nseg)
    kd = torch.from_numpy(k.view(np.int64).copy()).to(DEV)
    vd = torch.from_numpy(v.view(np.int32).copy()).to(DEV)
    bf.sort_u64(kd, vd, nseg=nseg)
    gk = kd.cpu().numpy().view(np.uint64).reshape(nseg, n)
    gv = vd.cpu().numpy().view(np.uint32).reshape(nseg, n)
    for s in range(nseg):
        seg = k[s * n:(s + 1) * n]
        order = np.argsort(seg, kind="stable")
        assert np.array_equal(gk[s], seg[order])
        assert np.array_equal(gv[s], order.astype(np.uint32))   # stable: equal keys keep their order


def test_radix_sort_keys_only():
    rng = np.random.default_rng(7)
    k = _keys(rng, 300_001, "doubles")
    kd = torch.from_numpy(k.view(np.int64).copy()).to(DEV)
    bf.sort_u64(kd)
    assert np.array_equal(kd.cpu().numpy().view(np.uint64), np.sort(k))


@pytest.mark.parametrize("n", [1, 7, 2048, 8192, 8193, 100_000, 3_000_001])
@pytest.mark.parametrize("inclusive", [False, True])
def test_scan_u32(n, inclusive):
    rng = np.random.default_rng(n)
    x = rng.integers(0, 1000, n).astype(np.uint32)
    g = bf.scan_u32(torch.from_numpy(x.view(np.int32)).to(DEV), inclusive).cpu().numpy().view(np.uint32)
    c = np.cumsum(x, dtype=np.uint64).astype(np.uint32)
    exp = c if inclusive else np.concatenate([[0], c[:-1]]).astype(np.uint32)
    assert np.array_equal(g, exp)


@pytest.mark.parametrize("n", [1, 5, 4096, 250_000])
def test_unique_u64(n):
    rng = np.random.default_rng(n)
    k = np.sort(_keys(rng, n, "ties"))
    u, cnt = bf.unique_u64(torch.from_numpy(k.view(np.int64)).to(DEV))
    ref = np.unique(k)
    assert cnt == ref.size and np.array_equal(u.cpu().numpy().view(np.uint64), ref)
