"""B200-native BlackForest random-forest hot path -- Python binding.

Thin ctypes marshalling over the C ABI of ``include/bf.h`` (``libbf.so``,
built from ``csrc/`` for sm_100a).  Every step of the method runs in the CUDA
kernels of that library; this module only converts torch tensors / numpy
arrays to pointers.  There is no CPU fallback: if the library is missing or
no CUDA device is present, the calls raise.

Matrices are column-major n x p, passed as (p, n) C-contiguous arrays
(``X[j, i]`` = predictor j of observation i).
"""
from __future__ import annotations

import ctypes as C
import os

import numpy as np

from . import build as _build

__all__ = ["Params", "Forest", "fit", "predict", "pca", "importance_finalize", "lib", "BFError"]

_LIB = None


class BFError(RuntimeError):
    def __init__(self, code: int, what: str, msg: str):
        super().__init__(f"{what} failed ({code}): {msg}")
        self.code = code


class Params(C.Structure):
    _fields_ = [
        ("ntree", C.c_int32), ("mtry", C.c_int32), ("nodesize", C.c_int32), ("replace", C.c_int32),
        ("sampsize", C.c_int64), ("seed", C.c_uint64), ("tree_begin", C.c_int32), ("tree_end", C.c_int32),
        ("trees_in_flight", C.c_int32), ("small_node_max", C.c_int32),
    ]


class Info(C.Structure):
    _fields_ = [
        ("n", C.c_int64), ("p", C.c_int32), ("ntree_total", C.c_int32), ("tree_begin", C.c_int32),
        ("tree_end", C.c_int32), ("total_nodes", C.c_int64), ("q", C.c_int32), ("mtry", C.c_int32),
        ("nodesize", C.c_int32), ("replace", C.c_int32), ("sampsize", C.c_int64), ("seed", C.c_uint64),
    ]


class View(C.Structure):
    _fields_ = [
        ("info", Info), ("tree_off", C.c_void_p), ("feature", C.c_void_p), ("left", C.c_void_p),
        ("thr_or_value", C.c_void_p), ("count", C.c_void_p), ("value", C.c_void_p), ("drss", C.c_void_p),
    ]


class Accum(C.Structure):
    _fields_ = [("d_slots", C.c_void_p), ("npur_slots", C.c_void_p), ("oob_sum", C.c_void_p),
                ("oob_cnt", C.c_void_p), ("e_t", C.c_void_p), ("nout_t", C.c_void_p)]


def lib():
    """Load libbf.so (building it with nvcc if it is absent or stale)."""
    global _LIB
    if _LIB is None:
        path = _build.LIB
        if not os.path.exists(path) or _build._stale():
            path = _build.build()
        L = C.CDLL(path, mode=C.RTLD_GLOBAL)
        vp, i32, i64, u64 = C.c_void_p, C.c_int32, C.c_int64, C.c_uint64
        sig = {
            "bf_version": ([], C.c_char_p), "bf_last_error": ([], C.c_char_p),
            "bf_fit": ([vp, i64, vp, i64, i32, C.POINTER(Params), vp, C.POINTER(vp)], C.c_int),
            "bf_forest_free": ([vp], None),
            "bf_forest_info_get": ([vp, C.POINTER(Info)], C.c_int),
            "bf_forest_export": ([vp, C.POINTER(View)], C.c_int),
            "bf_forest_import": ([C.POINTER(View), vp, C.POINTER(vp)], C.c_int),
            "bf_predict": ([vp, vp, i64, i64, vp, vp, i32, vp], C.c_int),
            "bf_oob_importance": ([vp, vp, i64, vp, i64, i32, C.POINTER(Accum), vp], C.c_int),
            "bf_importance_finalize": ([vp] * 5 + [i64, i32, i32] + [vp] * 6 + [vp], C.c_int),
            "bf_pca": ([vp, i64, i64, i32, i32, i32, vp, vp, vp, vp, vp], C.c_int),
            "bf_pca_retained": ([vp, i32, C.c_double, i32, vp, vp], C.c_int),
            "bf_partial_dependence": ([vp, vp, i64, i64, i32, i32, vp, i32, vp, vp, i32, vp], C.c_int),
            "bf_pd_grid": ([vp, i64, i32, vp, C.POINTER(C.c_int32), vp], C.c_int),
            "bf_varimax": ([vp, i64, i32, i32, i32, C.c_double, vp, vp, C.POINTER(C.c_int32), vp], C.c_int),
            "bf_glm_gaussian": ([vp, i64, i64, i32, vp, i64, i32, vp, vp, vp, vp], C.c_int),
            "bf_rank_similarity": ([vp, vp, i32, vp, vp], C.c_int),
            "bf_log_size_design": ([vp, i64, vp, i64, vp], C.c_int),
            "bf_prediction_error": ([vp, vp, i64, vp, vp], C.c_int),
            "bf_glm_predict": ([vp, i64, i64, i32, vp, i32, vp, i64, vp], C.c_int),
            "bf_mars_fit": ([vp, i64, i64, i32, vp, i32, C.c_double, C.c_double, C.POINTER(C.c_int32), vp, vp, vp, vp,
                             vp, vp], C.c_int),
            "bf_mars_predict": ([vp, i64, i64, i32, i32, vp, vp, vp, vp, vp, vp], C.c_int),
            "bf_philox": ([vp, C.c_uint32, C.c_uint32, vp, i64, vp], C.c_int),
            "bf_i128_to_double": ([vp, vp, vp, i64, vp], C.c_int),
            "bf_fixed_point": ([vp, i64, i64, vp, C.POINTER(C.c_int32), vp], C.c_int),
            "bf_bootstrap": ([u64, i32, i32, i64, i64, i32, vp, vp], C.c_int),
            "bf_perm": ([u64, i32, i32, i64, vp, vp], C.c_int),
            "bf_sort_u64": ([vp, vp, i64, i32, vp], C.c_int),
            "bf_scan_u32": ([vp, vp, i64, i32, vp], C.c_int),
            "bf_unique_u64": ([vp, i64, vp, vp, vp], C.c_int),
            "bf_set_allocator": ([vp, vp, vp], C.c_int),
            "bf_set_memory_budget": ([i64], C.c_int),
            "bf_release_workspace": ([], C.c_int),
            "bf_profile_enable": ([C.c_int], C.c_int),
            "bf_profile_read": ([vp, C.c_int, C.POINTER(C.c_int)], C.c_int),
            "bf_launch_count": ([], C.c_int64),
        }
        for name, (args, res) in sig.items():
            fn = getattr(L, name)
            fn.argtypes = args
            fn.restype = res
        _LIB = L
        _install_torch_allocator(L)
    return _LIB


_TORCH_ALLOC = None


def _install_torch_allocator(L):
    """Route every device allocation of libbf.so through torch's CUDA caching allocator (bf_set_allocator with
    the hooks of libbf_torch_alloc.so), so the library and the caller's tensors share one memory pool.
    Skipped without a CUDA device (nothing is allocated then) or with BF_TORCH_ALLOCATOR=0 (the library's own
    cudaMallocAsync pool)."""
    global _TORCH_ALLOC
    if os.environ.get("BF_TORCH_ALLOCATOR", "1") == "0":
        return
    torch = _torch()
    if not torch.cuda.is_available():
        return
    path = _build.TORCH_ALLOC
    if not os.path.exists(path) or os.path.getmtime(path) < os.path.getmtime(os.path.join(_build.CSRC, "torch_alloc.cpp")):
        path = _build.build_torch_alloc()
    A = C.CDLL(path)
    fa = C.cast(A.bf_torch_alloc, C.c_void_p).value
    ff = C.cast(A.bf_torch_free, C.c_void_p).value
    _check(L.bf_set_allocator(fa, ff, None), "bf_set_allocator")
    _TORCH_ALLOC = A


def torch_allocator_active() -> bool:
    lib()  # the hooks are installed when the library is loaded
    return _TORCH_ALLOC is not None


def _memory_budget_hint():
    """Free device memory as torch sees it (driver-free + torch-cached-but-unused blocks): bf_fit sizes its trees
    in flight from it when the torch allocator is installed."""
    if _TORCH_ALLOC is None:
        return
    torch = _torch()
    free, _ = torch.cuda.mem_get_info()
    lib().bf_set_memory_budget(int(free + torch.cuda.memory_reserved() - torch.cuda.memory_allocated()))


def exported_symbols():
    return [n for n in ("bf_version", "bf_last_error", "bf_set_allocator", "bf_set_memory_budget", "bf_release_workspace", "bf_fit", "bf_forest_free",
                        "bf_forest_info_get", "bf_forest_export", "bf_forest_import", "bf_predict",
                        "bf_oob_importance", "bf_importance_finalize", "bf_pca", "bf_pca_retained", "bf_philox", "bf_i128_to_double",
                        "bf_fixed_point", "bf_bootstrap", "bf_perm", "bf_sort_u64", "bf_scan_u32", "bf_unique_u64", "bf_profile_enable", "bf_profile_read",
                        "bf_launch_count", "bf_partial_dependence", "bf_pd_grid", "bf_varimax",
                        "bf_glm_gaussian", "bf_glm_predict", "bf_rank_similarity", "bf_log_size_design", "bf_prediction_error", "bf_mars_fit",
                        "bf_mars_predict")]


class KernelStat(C.Structure):
    _fields_ = [("name", C.c_char * 40), ("ms", C.c_double), ("launches", C.c_int64), ("bytes", C.c_double)]


def profile_enable(on: bool = True):
    lib().bf_profile_enable(int(on))


def profile_read() -> dict:
    """{kernel class: dict(ms, launches, bytes)} accumulated since the last read."""
    cnt = C.c_int()
    lib().bf_profile_read(None, 0, C.byref(cnt))  # size query drains nothing extra: totals are kept
    buf = (KernelStat * max(cnt.value + 64, 64))()
    lib().bf_profile_read(buf, len(buf), C.byref(cnt))
    return {buf[i].name.decode(): dict(ms=buf[i].ms, launches=int(buf[i].launches), bytes=buf[i].bytes)
            for i in range(min(cnt.value, len(buf)))}


def release_workspace() -> None:
    """Release the node-list work space bf_fit keeps across calls (bf_release_workspace)."""
    _check(lib().bf_release_workspace(), "bf_release_workspace")


def launch_count() -> int:
    return int(lib().bf_launch_count())


def _check(rc: int, what: str):
    if rc != 0:
        raise BFError(rc, what, lib().bf_last_error().decode())


def _torch():
    import torch
    return torch


def _ptr(a) -> int:
    """Data pointer of a torch tensor (CUDA or CPU) or a numpy array."""
    if isinstance(a, np.ndarray):
        if not a.flags.c_contiguous:
            raise ValueError("array must be C-contiguous")
        return a.ctypes.data
    if not a.is_contiguous():
        raise ValueError("tensor must be contiguous")
    return a.data_ptr()


def _stream(dev_like=None) -> int:
    torch = _torch()
    if torch.cuda.is_available():
        return torch.cuda.current_stream().cuda_stream
    return 0


def _is_cuda(a) -> bool:
    return not isinstance(a, np.ndarray) and a.is_cuda


def _empty_like_dev(ref, shape, dtype):
    """Output buffer on the same side (device tensor / host numpy) as ref."""
    torch = _torch()
    if _is_cuda(ref):
        tdt = {np.float64: torch.float64, np.int32: torch.int32, np.int64: torch.int64, np.uint32: torch.int32}[dtype]
        return torch.empty(shape, dtype=tdt, device=ref.device)
    return np.empty(shape, dtype=dtype)


class Forest:
    """Library-owned device forest for global trees [tree_begin, tree_end)."""

    def __init__(self, handle: C.c_void_p):
        self._h = handle

    def __del__(self):
        self.free()

    def free(self):
        if getattr(self, "_h", None):
            lib().bf_forest_free(self._h)
            self._h = None

    @property
    def info(self) -> Info:
        inf = Info()
        _check(lib().bf_forest_info_get(self._h, C.byref(inf)), "bf_forest_info_get")
        return inf

    def export(self) -> dict:
        """Host numpy arrays of the whole forest (see bf_forest_view)."""
        inf = self.info
        nt = inf.tree_end - inf.tree_begin
        tot = inf.total_nodes
        out = dict(tree_off=np.empty(nt + 1, np.int64), feature=np.empty(tot, np.int32), left=np.empty(tot, np.int32),
                   thr_or_value=np.empty(tot, np.float64), count=np.empty(tot, np.int32),
                   value=np.empty(tot, np.float64), drss=np.empty(tot, np.float64))
        v = View()
        for k in ("tree_off", "feature", "left", "thr_or_value", "count", "value", "drss"):
            setattr(v, k, out[k].ctypes.data if out[k].size else None)
        if out["tree_off"].size:
            v.tree_off = out["tree_off"].ctypes.data
        _check(lib().bf_forest_export(self._h, C.byref(v)), "bf_forest_export")
        out["info"] = inf
        return out

    def tree(self, i: int) -> dict:
        e = self.export() if not hasattr(self, "_export_cache") else self._export_cache
        self._export_cache = e
        lo, hi = e["tree_off"][i], e["tree_off"][i + 1]
        return {k: e[k][lo:hi] for k in ("feature", "left", "thr_or_value", "count", "value", "drss")}

    def predict(self, Xq, ntree_total: int = 0, out_sum=None, out_mean=None):
        """Returns (yhat_sum, yhat) as device tensors (device Xq) or numpy (host Xq)."""
        p, m = Xq.shape
        ys = _empty_like_dev(Xq, (m,), np.float64) if out_sum is None else out_sum
        yh = _empty_like_dev(Xq, (m,), np.float64) if out_mean is None else out_mean
        _check(lib().bf_predict(self._h, _ptr(Xq), m, m, _ptr(ys), _ptr(yh), ntree_total, _stream()), "bf_predict")
        return ys, yh

    def partial_dependence(self, X, m: int, grid=None, n_pt: int = 51, ntree_total: int = 0):
        """Partial dependence of the response on predictor m (bf_partial_dependence).
        X: (p, n) rows to average over.  grid: G values (default bf_pd_grid of X[m], n_pt points).
        Returns (grid, pd_sum, pd) on X's side (device tensors or numpy)."""
        p, n = X.shape
        if grid is None:
            grid = pd_grid(X[m], n_pt)
        G = int(grid.shape[0])
        ps = _empty_like_dev(X, (G,), np.float64)
        pd = _empty_like_dev(X, (G,), np.float64)
        _check(lib().bf_partial_dependence(self._h, _ptr(X), n, n, p, m, _ptr(grid), G, _ptr(ps), _ptr(pd),
                                           ntree_total, _stream()), "bf_partial_dependence")
        return grid, ps, pd

    def oob_importance(self, X, y, out: dict | None = None) -> dict:
        p, n = X.shape
        inf = self.info
        nt = inf.tree_end - inf.tree_begin
        if out is None:
            out = dict(d_slots=_empty_like_dev(X, (nt, p), np.float64), npur_slots=_empty_like_dev(X, (nt, p), np.float64),
                       oob_sum=_empty_like_dev(X, (n,), np.float64), oob_cnt=_empty_like_dev(X, (n,), np.int32),
                       e_t=_empty_like_dev(X, (max(nt, 1),), np.float64),
                       nout_t=_empty_like_dev(X, (max(nt, 1),), np.int64))
        acc = Accum(*[_ptr(out[k]) for k in ("d_slots", "npur_slots", "oob_sum", "oob_cnt", "e_t", "nout_t")])
        _check(lib().bf_oob_importance(self._h, _ptr(X), n, _ptr(y), n, p, C.byref(acc), _stream()),
               "bf_oob_importance")
        return out


def fit(X, y, ntree: int = 500, mtry: int = 0, nodesize: int = 5, replace: int = 1, sampsize: int = 0,
        seed: int = 0, tree_begin: int = 0, tree_end: int | None = None, trees_in_flight: int = 0,
        small_node_max: int = 0) -> Forest:
    """Grow global trees [tree_begin, tree_end).  X: (p, n) float64, y: (n,)."""
    p, n = X.shape
    prm = Params(ntree=ntree, mtry=mtry, nodesize=nodesize, replace=replace, sampsize=sampsize, seed=seed,
                 tree_begin=tree_begin, tree_end=ntree if tree_end is None else tree_end,
                 trees_in_flight=trees_in_flight, small_node_max=small_node_max)
    h = C.c_void_p()
    L = lib()
    _memory_budget_hint()
    _check(L.bf_fit(_ptr(X), n, _ptr(y), n, p, C.byref(prm), _stream(), C.byref(h)), "bf_fit")
    return Forest(h)


def forest_import(arrays: dict, info: Info) -> Forest:
    """Build a device forest from flat arrays (host numpy or device tensors)."""
    v = View()
    v.info = info
    for k in ("tree_off", "feature", "left", "thr_or_value", "count", "value", "drss"):
        a = arrays.get(k)
        setattr(v, k, _ptr(a) if a is not None and (a.size if isinstance(a, np.ndarray) else a.numel()) else None)
    if v.tree_off is None:
        raise ValueError("tree_off required")
    h = C.c_void_p()
    _check(lib().bf_forest_import(C.byref(v), _stream(), C.byref(h)), "bf_forest_import")
    return Forest(h)


def predict(forest: Forest, Xq, ntree_total: int = 0):
    return forest.predict(Xq, ntree_total)


def importance_finalize(d_slots, npur_slots, oob_sum, oob_cnt, y) -> dict:
    T, p = d_slots.shape
    n = y.shape[0]
    outs = {k: _empty_like_dev(y, (p,), np.float64) for k in ("inc_mse", "inc_mse_raw", "inc_mse_sd", "inc_node_purity")}
    sc = _empty_like_dev(y, (2,), np.float64)
    base = _ptr(sc)
    _check(lib().bf_importance_finalize(_ptr(d_slots), _ptr(npur_slots), _ptr(oob_sum), _ptr(oob_cnt), _ptr(y), n, p, T,
                                        _ptr(outs["inc_mse"]), _ptr(outs["inc_mse_raw"]), _ptr(outs["inc_mse_sd"]),
                                        _ptr(outs["inc_node_purity"]), base, base + 8, _stream()),
           "bf_importance_finalize")
    outs["oob_mse"] = sc[0]
    outs["rsq"] = sc[1]
    return outs


def pd_grid(x, n_pt: int = 51):
    """Default partial-dependence grid of one predictor column (bf_pd_grid, reading R23)."""
    n = int(x.shape[0])
    buf = _empty_like_dev(x, (n_pt,), np.float64)
    G = C.c_int32()
    xx = x if (isinstance(x, np.ndarray) and x.flags.c_contiguous) or (not isinstance(x, np.ndarray) and x.is_contiguous()) \
        else (np.ascontiguousarray(x) if isinstance(x, np.ndarray) else x.contiguous())
    _check(lib().bf_pd_grid(_ptr(xx), n, n_pt, _ptr(buf), C.byref(G), _stream()), "bf_pd_grid")
    return buf[: G.value]


def varimax(L, normalize: bool = True, eps: float = 1e-5) -> dict:
    """Varimax rotation of p x k loadings (bf_varimax, reading R25).  L: (k, p) array/tensor = column-major
    p x k.  Returns loadings (k, p), rotmat (k, k) (column-major k x k as (k, k) row blocks) and iterations."""
    k, p = L.shape
    lo = _empty_like_dev(L, (k, p), np.float64)
    ro = _empty_like_dev(L, (k, k), np.float64)
    it = C.c_int32()
    _check(lib().bf_varimax(_ptr(L), p, p, k, int(normalize), float(eps), _ptr(lo), _ptr(ro), C.byref(it),
                            _stream()), "bf_varimax")
    return {"loadings": lo, "rotmat": ro, "iters": int(it.value)}


def glm_gaussian(Z, Y) -> dict:
    """Counter models (bf_glm_gaussian, reading R26): Z (k, n) design = column-major n x k, Y (r, n) responses.
    Returns coef (r, k) (row j = coefficients of response j), deviance (r), null_deviance (r)."""
    k, n = Z.shape
    Y2 = Y.reshape(1, -1) if len(Y.shape) == 1 else Y
    r = Y2.shape[0]
    coef = _empty_like_dev(Z, (r, k), np.float64)
    dev = _empty_like_dev(Z, (r,), np.float64)
    nul = _empty_like_dev(Z, (r,), np.float64)
    _check(lib().bf_glm_gaussian(_ptr(Z), n, n, k, _ptr(Y2), n, r, _ptr(coef), _ptr(dev), _ptr(nul), _stream()),
           "bf_glm_gaussian")
    return {"coef": coef, "deviance": dev, "null_deviance": nul}


def glm_predict(Z, coef):
    """Counter models on new rows (bf_glm_predict): Z (k, n) design, coef (r, k).  Returns (r, n)."""
    k, n = Z.shape
    r = coef.shape[0]
    out = _empty_like_dev(Z, (r, n), np.float64)
    _check(lib().bf_glm_predict(_ptr(Z), n, n, k, _ptr(coef), r, _ptr(out), n, _stream()), "bf_glm_predict")
    return out


def mars_fit(X, y, nk: int = 0, thresh: float = 0.001, penalty: float = 2.0) -> dict:
    """MARS model of one response on (d, n) predictors (bf_mars_fit, reading R28).  Returns terms
    [(var, knot, dir)] (dir 0 = intercept), coef (numpy), rss, gcv, rsq."""
    d, n = X.shape
    cap = 32
    nt = C.c_int32()
    tv = np.zeros(cap, np.int32)
    tk = np.zeros(cap, np.float64)
    td = np.zeros(cap, np.int32)
    cf = np.zeros(cap, np.float64)
    st = np.zeros(3, np.float64)
    _check(lib().bf_mars_fit(_ptr(X), n, n, d, _ptr(y), nk, float(thresh), float(penalty), C.byref(nt), _ptr(tv),
                             _ptr(tk), _ptr(td), _ptr(cf), _ptr(st), _stream()), "bf_mars_fit")
    k = nt.value
    return {"terms": [(int(tv[j]), float(tk[j]), int(td[j])) for j in range(k)], "coef": cf[:k].copy(),
            "rss": float(st[0]), "gcv": float(st[1]), "rsq": float(st[2]),
            "_arrays": (tv[:k].copy(), tk[:k].copy(), td[:k].copy(), cf[:k].copy())}


def mars_predict(model: dict, X):
    """A bf_mars_fit model on new (d, m) rows (bf_mars_predict)."""
    d, m = X.shape
    tv, tk, td, cf = model["_arrays"]
    out = _empty_like_dev(X, (m,), np.float64)
    _check(lib().bf_mars_predict(_ptr(X), m, m, d, len(tv), _ptr(tv), _ptr(tk), _ptr(td), _ptr(cf), _ptr(out),
                                 _stream()), "bf_mars_predict")
    return out


def rank_similarity(a, b) -> tuple:
    """(Spearman rho, Kendall tau-b) of two importance vectors (bf_rank_similarity, reading R27)."""
    p = int(a.shape[0])
    out = _empty_like_dev(a, (2,), np.float64)
    _check(lib().bf_rank_similarity(_ptr(a), _ptr(b), p, _ptr(out), _stream()), "bf_rank_similarity")
    o = out.cpu().numpy() if hasattr(out, "cpu") else out
    return float(o[0]), float(o[1])


def pca(X, scale: bool = True, k: int | None = None) -> dict:
    """S9 PCA of (p, n) counters.  Returns sdev (p), rotation ((p, p): row j =
    component j, i.e. the column-major p x p matrix), center (p), scores ((k, n))."""
    p, n = X.shape
    kk = p if k is None else k
    sdev = _empty_like_dev(X, (p,), np.float64)
    rot = _empty_like_dev(X, (p, p), np.float64)
    cen = _empty_like_dev(X, (p,), np.float64)
    sco = _empty_like_dev(X, (max(kk, 1), n), np.float64)
    _check(lib().bf_pca(_ptr(X), n, n, p, int(scale), kk, _ptr(sdev), _ptr(rot), _ptr(cen), _ptr(sco), _stream()),
           "bf_pca")
    return dict(sdev=sdev, rotation=rot, center=cen, scores=sco[:kk])


def log_size_design(size):
    """[1, u, u^2, u^3] with u the standardised log2 of the sizes (bf_log_size_design, reading R26) -> (4, n)."""
    n = int(size.shape[0])
    Z = _empty_like_dev(size, (4, n), np.float64)
    _check(lib().bf_log_size_design(_ptr(size), n, _ptr(Z), n, _stream()), "bf_log_size_design")
    return Z


def prediction_error(yhat, y) -> tuple:
    """(mse, variance explained) of predicted times (bf_prediction_error)."""
    out = (C.c_double * 2)()
    _check(lib().bf_prediction_error(_ptr(yhat), _ptr(y), int(y.shape[0]), C.addressof(out), _stream()),
           "bf_prediction_error")
    return float(out[0]), float(out[1])


def pca_retained(sdev, frac: float = 0.97, cap: int = 10) -> int:
    """Number of retained components (bf_pca_retained, reading R15) from bf_pca's sdev."""
    k = C.c_int32()
    _check(lib().bf_pca_retained(_ptr(sdev), int(sdev.shape[0]), float(frac), int(cap), C.addressof(k), _stream()),
           "bf_pca_retained")
    return int(k.value)


# --- single-step entry points (parity tests) ---------------------------------

def philox(ctr: np.ndarray, key0: int, key1: int) -> np.ndarray:
    ctr = np.ascontiguousarray(ctr, np.uint32).reshape(-1, 4)
    out = np.empty_like(ctr)
    _check(lib().bf_philox(ctr.ctypes.data, key0, key1, out.ctypes.data, ctr.shape[0], _stream()), "bf_philox")
    return out


def sort_u64(keys, vals=None, nseg: int = 1):
    """In-place stable radix sort of device tensors (int64 storage of uint64 keys; int32 storage of uint32
    values) in nseg equal segments (bf_sort_u64)."""
    n = keys.numel() // nseg
    _check(lib().bf_sort_u64(_ptr(keys), _ptr(vals) if vals is not None else None, n, nseg, _stream()), "bf_sort_u64")


def scan_u32(x, inclusive: bool = False):
    """Prefix sum of a device int32 tensor holding uint32 values (bf_scan_u32)."""
    out = _torch().empty_like(x)
    _check(lib().bf_scan_u32(_ptr(x), _ptr(out), x.numel(), int(inclusive), _stream()), "bf_scan_u32")
    return out


def unique_u64(sorted_keys):
    """Distinct values of sorted device keys (bf_unique_u64) -> (values, count)."""
    torch = _torch()
    out = torch.empty_like(sorted_keys)
    cnt = torch.zeros(1, dtype=torch.int32, device=sorted_keys.device)
    _check(lib().bf_unique_u64(_ptr(sorted_keys), sorted_keys.numel(), _ptr(out), _ptr(cnt), _stream()), "bf_unique_u64")
    k = int(cnt.item())
    return out[:k], k


def i128_to_double(hi: np.ndarray, lo: np.ndarray) -> np.ndarray:
    hi = np.ascontiguousarray(hi, np.int64)
    lo = np.ascontiguousarray(lo, np.uint64)
    out = np.empty(hi.shape[0], np.float64)
    _check(lib().bf_i128_to_double(hi.ctypes.data, lo.ctypes.data, out.ctypes.data, hi.shape[0], _stream()),
           "bf_i128_to_double")
    return out


def fixed_point(y, sampsize: int = 0):
    n = y.shape[0]
    yq = _empty_like_dev(y, (n,), np.int64)
    q = C.c_int32()
    _check(lib().bf_fixed_point(_ptr(y), n, sampsize, _ptr(yq), C.byref(q), _stream()), "bf_fixed_point")
    return yq, int(q.value)


def bootstrap(seed: int, t0: int, ntrees: int, n: int, sampsize: int = 0, replace: int = 1) -> np.ndarray:
    w = np.empty((ntrees, n), np.int32)
    _check(lib().bf_bootstrap(seed, t0, ntrees, n, sampsize, replace, w.ctypes.data, _stream()), "bf_bootstrap")
    return w


def perm(seed: int, t: int, m: int, n_o: int) -> np.ndarray:
    out = np.empty(n_o, np.int64)
    _check(lib().bf_perm(seed, t, m, n_o, out.ctypes.data, _stream()), "bf_perm")
    return out
