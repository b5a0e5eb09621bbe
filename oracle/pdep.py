"""CPU ORACLE -- partial dependence.

TEST INFRASTRUCTURE ONLY (see oracle/oracle.py header).

PAPER.md:130 (sec 4.1.1): "the partial dependence plot, shows how the
response changes as a predictor or a set of predictors change(s)";
PAPER.md:165 (sec 5): "the partial dependence plot of the variable vis-a-vis
the execution time ... on the entire range of runs".  The paper names R
randomForest, whose partialPlot averages the forest prediction over
the training rows with the predictor set to each grid value.  Plain
definition (readings R23, R24):

  grid (R23): G = min(n_pt, #distinct x_m), v_g = lo + g * ((hi - lo)/(G-1)),
              v_{G-1} = hi (G = 1: v_0 = lo), lo/hi = min/max of x_m
  pd_sum[g] = sum_i sum_t f_t(x_i with x_im := v_g)     (oracle predict_sum)
  pd[g]     = pd_sum[g] / (n * T)                        (R24)
"""
from __future__ import annotations

import numpy as np


def pd_grid(x: np.ndarray, n_pt: int = 51) -> np.ndarray:
    x = np.asarray(x, dtype=np.float64) + 0.0  # -0.0 -> +0.0 (reading R18)
    G = min(int(n_pt), int(np.unique(x).shape[0]))
    lo, hi = float(x.min()), float(x.max())
    if G == 1:
        return np.array([lo])
    by = (hi - lo) / (G - 1)
    v = np.array([lo + g * by for g in range(G)], dtype=np.float64)
    v[-1] = hi
    return v


def partial_dependence(forest, X: np.ndarray, m: int, grid: np.ndarray, ntree_total: int | None = None):
    """forest: oracle.Forest; X: (p, n) rows to average over.  Returns (pd_sum, pd)."""
    X = np.asarray(X, dtype=np.float64)
    p, n = X.shape
    T = ntree_total or forest.ntrees_local()
    pd_sum = np.empty(len(grid))
    for g, v in enumerate(grid):
        Xg = X.copy()
        Xg[m, :] = v
        pd_sum[g] = forest.predict_sum(Xg).sum()
    return pd_sum, pd_sum / (n * T)
