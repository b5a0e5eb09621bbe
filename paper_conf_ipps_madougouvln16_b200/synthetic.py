"""Seeded synthetic counter datasets shaped like the paper's use cases.

This module holds NO arithmetic of the method: it only draws inputs
(X, y, query rows) with numpy's Philox bit generator.  Both the CUDA path
(tests, bench) and the CPU oracle consume these arrays; neither side's code
lives here.

Recipe:
  * a hidden problem size drives everything ("running the
    application multiple times ... with different problem characteristics");
  * counters from Table 1: integer counts (lognormal, heavy
    right tail, many ties), ratios in (0, 1), throughputs > 0, all functions
    of a few latent factors plus noise ("four principal
    components ... more than 97% of the variance");
  * response = execution time > 0 with 2% lognormal noise;
  * at least one pure-noise U(0,1) column (the importance ~ 0 pin).

Arrays are returned as (p, n) C-contiguous float64 == column-major n x p,
the layout of the C-ABI (element (i, j) at X[j*n + i]).
"""
from __future__ import annotations

from dataclasses import dataclass, field

import numpy as np

DATA_SEED = 0xBF00_0000
FOREST_SEED = 0xBF10_0000
QUERY_SEED = 0xBF20_0000


@dataclass
class Config:
    name: str
    n: int
    p: int
    ntree: int
    mtry: int = 0          # 0 -> max(p // 3, 1)
    nodesize: int = 5
    m_query: int = 0       # query rows for predictions/s
    importance: bool = False
    pca: bool = False
    notes: str = ""
    extra: dict = field(default_factory=dict)


# BASELINE.json configs[0..4]
CONFIGS = {
    "C1": Config("C1-reduction", 256, 20, 500, m_query=1 << 20,
                 notes="reduce6-like: 256 runs x 20 counters"),
    "C2": Config("C2-matmul", 4096, 41, 500, importance=True, m_query=1 << 20,
                 notes="tiled MM: 64 sizes N in {32..2048} x 64 replicates; 40 counters + N"),
    "C3": Config("C3-nw-hwscaling", 16384, 60, 500, pca=True, m_query=1 << 20,
                 notes="NW: L in {64..8192 step 64} x 3 GPU generations; 60 counters -> PCA"),
    "C4": Config("C4-scaled", 1_000_000, 64, 1000, importance=True, pca=True, m_query=10_000_000,
                 notes="1M runs x 64 predictors (48 counters of 6 latents + 8 problem/machine + 8 noise)"),
}


def _rng(seed: int) -> np.random.Generator:
    return np.random.Generator(np.random.Philox(seed))


def _counter_block(rng, Z: np.ndarray, n_counters: int, kinds=("count", "ratio", "thru")) -> np.ndarray:
    """Counters as noisy monotone functions of latent factors Z (n x L)."""
    n, L = Z.shape
    out = np.empty((n_counters, n), np.float64)
    for j in range(n_counters):
        kind = kinds[j % len(kinds)]
        a = rng.normal(0.0, 1.0, L) * (rng.random(L) < 0.6)
        if not a.any():
            a[rng.integers(L)] = 1.0
        lin = Z @ a + rng.normal(0.0, 0.05, n)
        if kind == "count":
            scale = 10.0 ** rng.uniform(2, 8)
            out[j] = np.rint(scale * np.exp(0.8 * lin))           # integers: ties
        elif kind == "ratio":
            out[j] = 1.0 / (1.0 + np.exp(-lin))                    # in (0, 1)
        else:
            out[j] = 10.0 ** rng.uniform(0, 3) * np.exp(0.5 * lin)  # throughput > 0
    return out


def gen_reduction(n: int = 256, p: int = 20, seed: int = DATA_SEED + 1):
    """C1: reduction kernel runs, array length s = 2^u, u ~ U(10, 26)."""
    rng = _rng(seed)
    u = rng.uniform(10, 26, n)
    s = np.exp2(u)
    bw = 1.0 / (1.0 + np.exp(-(u - 16.0)))            # bandwidth saturates with size
    Z = np.stack([(u - 18) / 5, bw - 0.5, rng.normal(0, 1, n), rng.normal(0, 1, n)], axis=1)
    X = _counter_block(rng, Z, p - 1)
    X = np.concatenate([X, rng.random((1, n))], axis=0)  # pure-noise column last
    y = (s / (1e3 * (0.1 + bw)) + 5.0) * np.exp(0.02 * rng.normal(0, 1, n))
    return np.ascontiguousarray(X), y


def gen_mm(n: int = 4096, p: int = 41, seed: int = DATA_SEED + 2):
    """C2: tiled MM, N in {32, 64, ..., 2048} (PAPER.md:222 range 2^5..2^11) x replicates."""
    rng = _rng(seed)
    sizes = np.arange(32, 2049, 32, dtype=np.float64)
    N = sizes[np.arange(n) % len(sizes)]
    lg = np.log2(N)
    Z = np.stack([(lg - 8) / 2, ((lg - 8) / 2) ** 2, rng.normal(0, 0.3, n), rng.normal(0, 1, n)], axis=1)
    X = _counter_block(rng, Z, p - 2)
    X = np.concatenate([X, rng.random((1, n)), N[None, :]], axis=0)   # noise column, then N
    y = (2.0 * N ** 3 / 1e9 * (1.0 + 0.3 * np.tanh(Z[:, 2])) + 0.01) * np.exp(0.02 * rng.normal(0, 1, n))
    return np.ascontiguousarray(X), y


# Table 2: wsched, freq (GHz), smp (SMs), rco (cores/SM), mbw (GB/s), regs, L2 (KB);
# generation 3 values are ours.
MACHINES = np.array([
    [2, 1.401, 15, 32, 177.4, 63, 768],     # GTX480 (Fermi)
    [4, 0.706, 13, 192, 208.0, 255, 1536],  # K20m (Kepler)
    [4, 1.126, 16, 128, 224.0, 255, 2048],  # synthetic gen-3
], dtype=np.float64)


def gen_nw(n: int = 16384, n_counters: int = 60, seed: int = DATA_SEED + 3):
    """C3: NW, L uniform over {64..8192 step 64} x 3 generations.
    Returns counters (60, n), sequence length L (n), machine metrics (7, n), y."""
    rng = _rng(seed)
    L = 64.0 * rng.integers(1, 129, n)
    g = rng.integers(0, 3, n)
    M = MACHINES[g]                                   # n x 7
    lg = np.log2(L)
    cache = M[:, 6] / 2048.0
    Z = np.stack([(lg - 10) / 2, cache - 0.7, (M[:, 4] - 200) / 30, rng.normal(0, 1, n)], axis=1)
    X = _counter_block(rng, Z, n_counters)
    work = (L / 64.0) ** 2
    y = (work / (M[:, 2] * M[:, 3] * M[:, 1]) * (1.0 + 0.5 * (cache < 0.5)) + 0.05) * np.exp(
        0.02 * rng.normal(0, 1, n))
    return np.ascontiguousarray(X), L, np.ascontiguousarray(M.T), y


def gen_scaled(n: int = 1_000_000, seed: int = DATA_SEED + 4, chunk: int = 1 << 18):
    """C4: 64 predictors = 48 counters of 6 latent factors + 8 problem/machine + 8 noise;
    Friedman-1-like response on the latents.  Generated in chunks (fixed chunk seeds)."""
    p = 64
    X = np.empty((p, n), np.float64)
    y = np.empty(n, np.float64)
    coef_rng = _rng(seed)
    A = coef_rng.normal(0, 1, (6, 48)) * (coef_rng.random((6, 48)) < 0.5)
    A[coef_rng.integers(0, 6, 48), np.arange(48)] += 1.0
    kinds = np.arange(48) % 3
    scales = 10.0 ** coef_rng.uniform(2, 8, 48)
    for c0 in range(0, n, chunk):
        c1 = min(n, c0 + chunk)
        m = c1 - c0
        rng = _rng(seed + 0x1000 + c0 // chunk)
        U = rng.random((m, 6))
        Z = (U - 0.5) * 2.0
        lin = Z @ A + rng.normal(0, 0.05, (m, 48))
        cnt = np.rint(scales * np.exp(0.8 * lin))
        rat = 1.0 / (1.0 + np.exp(-lin))
        thr = 10.0 * np.exp(0.5 * lin)
        C = np.where(kinds == 0, cnt, np.where(kinds == 1, rat, thr))
        X[:48, c0:c1] = C.T
        size = np.exp2(np.floor(10 + 16 * U[:, 0]))                  # problem size (integer, ties)
        X[48, c0:c1] = size
        X[49:56, c0:c1] = MACHINES[rng.integers(0, 3, m)].T
        X[56:64, c0:c1] = rng.random((8, m))                          # pure noise
        f1 = 10 * np.sin(np.pi * U[:, 0] * U[:, 1]) + 20 * (U[:, 2] - 0.5) ** 2 + 10 * U[:, 3] + 5 * U[:, 4]
        y[c0:c1] = (f1 + 5.0) * np.exp(0.02 * rng.normal(0, 1, m))
    return X, y


def gen_query(X: np.ndarray, m: int, seed: int = QUERY_SEED, chunk: int = 1 << 20) -> np.ndarray:
    """Query rows: resample training rows column-wise-jointly and jitter the
    continuous values (keeps each counter's distribution and ties)."""
    p, n = X.shape
    Q = np.empty((p, m), np.float64)
    for c0 in range(0, m, chunk):
        c1 = min(m, c0 + chunk)
        rng = _rng(seed + c0 // chunk)
        idx = rng.integers(0, n, c1 - c0)
        Q[:, c0:c1] = X[:, idx]
        jit = rng.random((p, c1 - c0)) < 0.5
        Q[:, c0:c1] = np.where(jit, Q[:, c0:c1] * (1.0 + 0.01 * rng.normal(0, 1, (p, c1 - c0))), Q[:, c0:c1])
    return Q


def dataset(cfg: str):
    """(X (p, n), y, Config) for C1..C4.  C3 returns the RF-input matrix
    [PC scores | L | 7 machine metrics] is assembled by the caller after PCA;
    here X = the 60 raw counters and extra = {L, M}."""
    c = CONFIGS[cfg]
    if cfg == "C1":
        X, y = gen_reduction(c.n, c.p)
    elif cfg == "C2":
        X, y = gen_mm(c.n, c.p)
    elif cfg == "C3":
        X, L, M, y = gen_nw(c.n, c.p)
        c.extra = dict(L=L, M=M)
    elif cfg == "C4":
        X, y = gen_scaled(c.n)
    else:
        raise KeyError(cfg)
    return X, y, c


def small_random(n: int, p: int, seed: int, kind: str = "mixed"):
    """Small random problems for parity tests: 'int' = small-integer x with
    many ties; 'cont' = continuous; 'mixed' = both; y continuous."""
    rng = _rng(seed)
    if kind == "int":
        X = rng.integers(0, 5, (p, n)).astype(np.float64)
    elif kind == "cont":
        X = rng.normal(0, 1, (p, n))
    else:
        X = np.where(rng.random((p, 1)) < 0.5, rng.integers(0, 8, (p, n)).astype(np.float64), rng.normal(0, 1, (p, n)))
    y = X[0] * 2.0 + np.sin(X[min(1, p - 1)]) + rng.normal(0, 0.3, n)
    return np.ascontiguousarray(X), y
