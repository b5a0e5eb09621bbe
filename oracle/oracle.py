"""CPU ORACLE -- ctypes wrapper around oracle/libbfo.so (oracle/bfo.c).

TEST INFRASTRUCTURE ONLY.  Only tests/, ``__graft_entry__.smoke()`` and the
``cpu_baseline`` / ``--impl reference`` legs of ``bench.py`` may import this
module.  The product package never imports anything under ``oracle/``.

The functions mirror the C-ABI of the product (``bf_*``) over host numpy
arrays with the ``bfo_`` prefix.  Semantics: DESIGN.md section 2 (S1..S9),
citing PAPER.md (P:71 learning set, P:75-95 trees and forest, P:130
permutation importance, P:157 OOB validation).
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "libbfo.so")
_SRC = os.path.join(_HERE, "bfo.c")


def build(force: bool = False) -> str:
    """Compile oracle/bfo.c with gcc (plain C11, no FMA contraction)."""
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < max(
        os.path.getmtime(_SRC), os.path.getmtime(os.path.join(_HERE, "bfo.h"))
    ):
        subprocess.check_call(
            ["gcc", "-O2", "-ffp-contract=off", "-std=gnu11", "-fPIC", "-shared",
             "-o", _SO, _SRC, "-lm", "-lpthread"]
        )
    return _SO


class Params(C.Structure):
    _fields_ = [
        ("ntree", C.c_int32), ("mtry", C.c_int32), ("nodesize", C.c_int32), ("replace", C.c_int32),
        ("sampsize", C.c_int64), ("seed", C.c_uint64), ("tree_begin", C.c_int32), ("tree_end", C.c_int32),
        ("nthreads", C.c_int32), ("pad_", C.c_int32),
    ]


_lib = None


def lib():
    global _lib
    if _lib is None:
        build()
        L = C.CDLL(_SO)
        P = C.POINTER
        L.bfo_philox4x32_10.argtypes = [P(C.c_uint32), P(C.c_uint32), P(C.c_uint32)]
        L.bfo_mulhi64.argtypes = [C.c_uint64, C.c_uint64]
        L.bfo_mulhi64.restype = C.c_uint64
        L.bfo_fixed_point.argtypes = [C.c_void_p, C.c_int64, C.c_int64, C.c_void_p, P(C.c_int32)]
        L.bfo_bootstrap.argtypes = [C.c_uint64, C.c_int32, C.c_int64, C.c_int64, C.c_int32, C.c_void_p]
        L.bfo_draw_mtry.argtypes = [C.c_uint64, C.c_int32, C.c_uint64, C.c_int32, C.c_int32, C.c_void_p]
        L.bfo_child_key.argtypes = [C.c_uint64, C.c_int32, C.c_uint64, C.c_int32]
        L.bfo_child_key.restype = C.c_uint64
        L.bfo_perm.argtypes = [C.c_uint64, C.c_int32, C.c_int32, C.c_int64, C.c_int64]
        L.bfo_perm.restype = C.c_int64
        L.bfo_i128_to_double.argtypes = [C.c_int64, C.c_uint64]
        L.bfo_i128_to_double.restype = C.c_double
        L.bfo_fit.argtypes = [C.c_void_p, C.c_int64, C.c_void_p, C.c_int64, C.c_int32, P(Params), P(C.c_void_p)]
        L.bfo_forest_free.argtypes = [C.c_void_p]
        L.bfo_forest_ntrees.argtypes = [C.c_void_p]
        L.bfo_forest_q.argtypes = [C.c_void_p]
        L.bfo_tree_nnodes.argtypes = [C.c_void_p, C.c_int32]
        L.bfo_tree_nnodes.restype = C.c_int64
        L.bfo_tree_export.argtypes = [C.c_void_p, C.c_int32] + [C.c_void_p] * 6
        L.bfo_predict.argtypes = [C.c_void_p, C.c_void_p, C.c_int64, C.c_int64, C.c_void_p]
        L.bfo_oob_importance.argtypes = [C.c_void_p, C.c_void_p, C.c_int64, C.c_void_p, C.c_int64, C.c_int32,
                                         C.c_int32] + [C.c_void_p] * 6
        L.bfo_importance_finalize.argtypes = [C.c_void_p] * 5 + [C.c_int64, C.c_int32, C.c_int32] + [C.c_void_p] * 6
        _lib = L
    return _lib


def _ptr(a: np.ndarray) -> int:
    return a.ctypes.data


class OracleError(RuntimeError):
    pass


def _check(rc: int, what: str):
    if rc != 0:
        raise OracleError(f"{what} failed with code {rc}")


# --- primitives -------------------------------------------------------------

def philox(ctr, key):
    c = (C.c_uint32 * 4)(*[int(v) & 0xFFFFFFFF for v in ctr])
    k = (C.c_uint32 * 2)(*[int(v) & 0xFFFFFFFF for v in key])
    o = (C.c_uint32 * 4)()
    lib().bfo_philox4x32_10(c, k, o)
    return [int(v) for v in o]


def mulhi64(u: int, r: int) -> int:
    return int(lib().bfo_mulhi64(u, r))


def fixed_point(y: np.ndarray, sampsize: int | None = None):
    y = np.ascontiguousarray(y, dtype=np.float64)
    yq = np.empty(y.shape[0], dtype=np.int64)
    q = C.c_int32()
    _check(lib().bfo_fixed_point(_ptr(y), y.shape[0], sampsize or y.shape[0], _ptr(yq), C.byref(q)), "fixed_point")
    return yq, int(q.value)


def bootstrap(seed: int, t: int, n: int, sampsize: int | None = None, replace: int = 1) -> np.ndarray:
    w = np.empty(n, dtype=np.int32)
    _check(lib().bfo_bootstrap(seed, t, n, sampsize or n, replace, _ptr(w)), "bootstrap")
    return w


def draw_mtry(seed: int, t: int, key: int, p: int, mtry: int) -> np.ndarray:
    f = np.empty(mtry, dtype=np.int32)
    lib().bfo_draw_mtry(seed, t, key, p, mtry, _ptr(f))
    return f


def child_key(seed: int, t: int, key: int, side: int) -> int:
    return int(lib().bfo_child_key(seed, t, key, side))


def perm(seed: int, t: int, m: int, n_o: int, a: int) -> int:
    return int(lib().bfo_perm(seed, t, m, n_o, a))


def i128_to_double(v: int) -> float:
    v &= (1 << 128) - 1
    hi = v >> 64
    if hi >= 1 << 63:
        hi -= 1 << 64
    return float(lib().bfo_i128_to_double(hi, v & ((1 << 64) - 1)))


# --- forest -----------------------------------------------------------------

class Forest:
    """Host-side oracle forest for global trees [tree_begin, tree_end)."""

    def __init__(self, handle, n, p, params: Params):
        self._h = handle
        self.n, self.p = n, p
        self.params = params
        self.ntree = params.ntree
        self.tree_begin, self.tree_end = params.tree_begin, params.tree_end

    def __del__(self):
        if getattr(self, "_h", None):
            lib().bfo_forest_free(self._h)
            self._h = None

    @property
    def q(self) -> int:
        return int(lib().bfo_forest_q(self._h))

    def ntrees_local(self) -> int:
        return int(lib().bfo_forest_ntrees(self._h))

    def tree(self, i: int) -> dict:
        """Local tree i in BFS order (dict of numpy arrays)."""
        nn = int(lib().bfo_tree_nnodes(self._h, i))
        d = dict(feature=np.empty(nn, np.int32), thr=np.empty(nn, np.float64), left=np.empty(nn, np.int32),
                 count=np.empty(nn, np.int64), value=np.empty(nn, np.float64), drss=np.empty(nn, np.float64))
        _check(lib().bfo_tree_export(self._h, i, _ptr(d["feature"]), _ptr(d["thr"]), _ptr(d["left"]),
                                     _ptr(d["count"]), _ptr(d["value"]), _ptr(d["drss"])), "tree_export")
        return d

    def predict_sum(self, Xq: np.ndarray) -> np.ndarray:
        """Sum over this forest's trees (column-major Xq given as (p, m) array)."""
        Xq = np.ascontiguousarray(Xq, dtype=np.float64)
        p, m = Xq.shape
        out = np.empty(m, np.float64)
        _check(lib().bfo_predict(self._h, _ptr(Xq), m, m, _ptr(out)), "predict")
        return out

    def oob_importance(self, X: np.ndarray, y: np.ndarray, perm_identity: bool = False) -> dict:
        X = np.ascontiguousarray(X, dtype=np.float64)
        y = np.ascontiguousarray(y, dtype=np.float64)
        p, n = X.shape
        nt = self.ntrees_local()
        r = dict(d_slots=np.zeros((nt, p)), npur_slots=np.zeros((nt, p)), oob_sum=np.zeros(n),
                 oob_cnt=np.zeros(n, np.int32), e_t=np.zeros(nt), nout_t=np.zeros(nt, np.int64))
        _check(lib().bfo_oob_importance(self._h, _ptr(X), n, _ptr(y), n, p, int(perm_identity),
                                        _ptr(r["d_slots"]), _ptr(r["npur_slots"]), _ptr(r["oob_sum"]),
                                        _ptr(r["oob_cnt"]), _ptr(r["e_t"]), _ptr(r["nout_t"])), "oob_importance")
        return r


def fit(X: np.ndarray, y: np.ndarray, ntree: int = 500, mtry: int = 0, nodesize: int = 5, replace: int = 1,
        sampsize: int = 0, seed: int = 0, tree_begin: int = 0, tree_end: int | None = None,
        nthreads: int = 1) -> Forest:
    """X given as a (p, n) C-contiguous array == column-major n x p."""
    X = np.ascontiguousarray(X, dtype=np.float64)
    y = np.ascontiguousarray(y, dtype=np.float64)
    p, n = X.shape
    prm = Params(ntree=ntree, mtry=mtry, nodesize=nodesize, replace=replace, sampsize=sampsize, seed=seed,
                 tree_begin=tree_begin, tree_end=ntree if tree_end is None else tree_end, nthreads=nthreads)
    h = C.c_void_p()
    _check(lib().bfo_fit(_ptr(X), n, _ptr(y), n, p, C.byref(prm), C.byref(h)), "fit")
    return Forest(h, n, p, prm)


def importance_finalize(d_slots, npur_slots, oob_sum, oob_cnt, y) -> dict:
    d_slots = np.ascontiguousarray(d_slots, np.float64)
    npur_slots = np.ascontiguousarray(npur_slots, np.float64)
    oob_sum = np.ascontiguousarray(oob_sum, np.float64)
    oob_cnt = np.ascontiguousarray(oob_cnt, np.int32)
    y = np.ascontiguousarray(y, np.float64)
    T, p = d_slots.shape
    n = y.shape[0]
    out = dict(inc_mse=np.empty(p), inc_mse_raw=np.empty(p), inc_mse_sd=np.empty(p), inc_node_purity=np.empty(p))
    mse = C.c_double()
    rsq = C.c_double()
    _check(lib().bfo_importance_finalize(_ptr(d_slots), _ptr(npur_slots), _ptr(oob_sum), _ptr(oob_cnt), _ptr(y),
                                         n, p, T, _ptr(out["inc_mse"]), _ptr(out["inc_mse_raw"]),
                                         _ptr(out["inc_mse_sd"]), _ptr(out["inc_node_purity"]),
                                         C.addressof(mse), C.addressof(rsq)), "importance_finalize")
    out["oob_mse"] = mse.value
    out["rsq"] = rsq.value
    return out
