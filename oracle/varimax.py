"""CPU ORACLE -- varimax rotation of PCA loadings.

TEST INFRASTRUCTURE ONLY (see oracle/oracle.py header).

PAPER.md:169 ("Refinement with PCA ... we use the factor loadings of the
variable with relation to the retained principal components"), P:134 and
P:177 (R toolchain: prcomp).  The rotation of the retained loadings is the
R stats ``varimax(x, normalize = TRUE, eps = 1e-5)`` iteration (reading R25),
restated step by step:

  if k < 2: return x, I
  if normalize: sc_i = sqrt(sum_j x_ij^2); x_ij = x_ij / sc_i
  T = I_k; d = 0
  repeat (at most 1000 times):
      Z = x T
      B = x^T (Z^3 - Z diag(sum_i Z_ij^2) / p)        (Z^3 elementwise)
      B = U diag(s) V^T                                 (library SVD)
      T = U V^T;  d_past = d;  d = sum(s)
      if d < d_past * (1 + eps): stop
  Z = x T; if normalize: Z_ij = Z_ij * sc_i
  return loadings Z, rotation T, iterations
"""
from __future__ import annotations

import numpy as np


def varimax(x: np.ndarray, normalize: bool = True, eps: float = 1e-5, max_iter: int = 1000):
    x = np.array(x, dtype=np.float64)
    p, k = x.shape
    if k < 2:
        return x, np.eye(k), 0
    sc = None
    if normalize:
        sc = np.sqrt((x * x).sum(axis=1))
        x = x / sc[:, None]
    T = np.eye(k)
    d = 0.0
    it = 0
    for it in range(1, max_iter + 1):
        Z = x @ T
        B = x.T @ (Z ** 3 - Z * ((Z ** 2).sum(axis=0) / p)[None, :])
        U, s, Vt = np.linalg.svd(B)
        T = U @ Vt
        d_past = d
        d = float(s.sum())
        if d < d_past * (1 + eps):
            break
    Z = x @ T
    if normalize:
        Z = Z * sc[:, None]
    return Z, T, it


def criterion(z: np.ndarray) -> float:
    """Raw varimax criterion sum_j [ sum_i z_ij^4 - (sum_i z_ij^2)^2 / p ]."""
    p = z.shape[0]
    return float(((z ** 4).sum(axis=0) - (z ** 2).sum(axis=0) ** 2 / p).sum())


def loadings_from_pca(rotation: np.ndarray, sdev: np.ndarray, k: int) -> np.ndarray:
    """Factor loadings of the first k components: rotation[:, j] * sdev[j] (reading R25)."""
    return rotation[:, :k] * sdev[None, :k]
