"""CPU ORACLE -- principal component analysis of counters (spec S9).

TEST INFRASTRUCTURE ONLY (see oracle/oracle.py header).

PAPER.md:134 (sec 4.1.2): "PCA produces new variables, called principal
components, from linear combinations of the original (potentially
correlated) variables such that there is no correlation between these
components"; PAPER.md:177 (sec 4.3): R ``prcomp``.  Plain definition in fp64:

  mu_j = column mean; if scale: sigma_j = sample sd (n-1), Z = (X-mu)/sigma
  C = Z^T Z / (n-1)                                    (library matmul)
  C = V diag(lambda) V^T, lambda descending            (numpy.linalg.eigh)
  sign rule: each column of V has its largest-|.| entry positive (ties ->
  lowest index)                                         (reading R16)
  sdev = sqrt(max(lambda, 0)); scores = Z V[:, :k]
"""
from __future__ import annotations

import numpy as np


def pca(X: np.ndarray, scale: bool = True, k: int | None = None) -> dict:
    """X: (p, n) array = column-major n x p counters.  Returns sdev (p),
    rotation (p x p, columns = components), scores (n x k)."""
    X = np.asarray(X, dtype=np.float64)
    p, n = X.shape
    if n < 2:
        raise ValueError("need n >= 2")
    Xt = X.T  # n x p view
    mu = Xt.mean(axis=0)
    Z = Xt - mu
    if scale:
        sd = np.sqrt((Z * Z).sum(axis=0) / (n - 1))
        if np.any(sd == 0.0):
            raise ValueError("constant column with scale=True")
        Z = Z / sd
    Cm = (Z.T @ Z) / (n - 1)
    lam, V = np.linalg.eigh(Cm)
    order = np.argsort(-lam, kind="stable")
    lam = lam[order]
    V = V[:, order]
    for j in range(p):
        col = V[:, j]
        i = int(np.argmax(np.abs(col)))  # first index of the max -> lowest on ties
        if col[i] < 0:
            V[:, j] = -col
    sdev = np.sqrt(np.maximum(lam, 0.0))
    kk = p if k is None else k
    scores = Z @ V[:, :kk]
    return dict(sdev=sdev, rotation=V, scores=scores, center=mu, cov=Cm)


def n_components(sdev: np.ndarray, frac: float = 0.97, cap: int = 10) -> int:
    """Reading R15: smallest k with cumulative variance >= frac, capped (P:134 '<10', P:189 '>97%')."""
    v = sdev ** 2
    c = np.cumsum(v) / v.sum()
    k = int(np.searchsorted(c, frac) + 1)
    return max(1, min(k, cap, len(sdev)))
