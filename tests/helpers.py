"""Shared test helpers: structural tree comparison GPU forest vs oracle forest."""
from __future__ import annotations

import numpy as np


def compare_tree(g: dict, o: dict, value_rtol: float = 1e-9, tag: str = "") -> int:
    """g: GPU tree (feature, left, thr_or_value, count, value, drss; any node
    order, root 0, right = left + 1).  o: oracle tree (BFS order).  Topology
    (feature, threshold, left/right structure, counts) must be bit-exact;
    node values within value_rtol (fp64 sums in a different order)."""
    stack = [(0, 0)]
    seen = 0
    while stack:
        kg, ko = stack.pop()
        seen += 1
        fg, fo = int(g["feature"][kg]), int(o["feature"][ko])
        assert fg == fo, f"{tag} feature mismatch gpu node {kg} ({fg}) vs oracle node {ko} ({fo})"
        assert int(g["count"][kg]) == int(o["count"][ko]), f"{tag} count mismatch at oracle node {ko}"
        ov = o["value"][ko]
        assert abs(g["value"][kg] - ov) <= value_rtol * max(abs(ov), 1e-300) + 1e-300, \
            f"{tag} value mismatch at oracle node {ko}: {g['value'][kg]!r} vs {ov!r}"
        if fo >= 0:
            tg = g["thr_or_value"][kg]
            assert tg == o["thr"][ko], f"{tag} threshold mismatch at oracle node {ko}: {tg!r} vs {o['thr'][ko]!r}"
            od = o["drss"][ko]
            assert abs(g["drss"][kg] - od) <= 1e-12 * abs(od) + 1e-300, f"{tag} drss mismatch at {ko}"
            lg, lo = int(g["left"][kg]), int(o["left"][ko])
            stack.append((lg, lo))
            stack.append((lg + 1, lo + 1))
        else:
            assert abs(g["thr_or_value"][kg] - ov) <= value_rtol * max(abs(ov), 1e-300) + 1e-300
    assert seen == len(o["feature"]), f"{tag} node count: walked {seen}, oracle has {len(o['feature'])}"
    assert seen == len(g["feature"]), f"{tag} node count: walked {seen}, gpu has {len(g['feature'])}"
    return seen


def compare_forest(gf, of, value_rtol: float = 1e-9, trees=None):
    e = gf.export()
    nt = len(e["tree_off"]) - 1
    assert nt == of.ntrees_local()
    total = 0
    for i in (range(nt) if trees is None else trees):
        lo, hi = e["tree_off"][i], e["tree_off"][i + 1]
        g = {k: e[k][lo:hi] for k in ("feature", "left", "thr_or_value", "count", "value", "drss")}
        total += compare_tree(g, of.tree(i), value_rtol, tag=f"tree {i}:")
    return total


def rel_close(a, b, rtol, atol_scale=0.0):
    a = np.asarray(a, np.float64)
    b = np.asarray(b, np.float64)
    scale = atol_scale * max(np.abs(b).max(initial=0.0), 1e-300)
    return np.all(np.abs(a - b) <= rtol * np.abs(b) + scale)


def assert_same_ranking(g, o, rtol: float = 1e-12, tag: str = ""):
    """Importance ranking identical (BASELINE north_star): every pair of predictors is ordered the
    same way by g (GPU) and o (oracle).  The only pairs allowed to differ are those whose OWN oracle
    values agree to within rtol * max|o| (a tie within rounding, reported in the message, not hidden)."""
    g = np.asarray(g, np.float64)
    o = np.asarray(o, np.float64)
    scale = rtol * max(np.abs(o).max(initial=0.0), 1e-300)
    sg = np.sign(g[:, None] - g[None, :])
    so = np.sign(o[:, None] - o[None, :])
    bad = np.argwhere((sg != so) & (np.abs(o[:, None] - o[None, :]) > scale))
    assert bad.size == 0, f"{tag} ranking differs for pairs {bad[:8].tolist()} (oracle {o}, gpu {g})"
    return int(np.count_nonzero(sg != so)) // 2


def eigen_clusters(lam, rel: float = 1e-6):
    """Groups of consecutive eigenvalues (descending) closer than rel * lam[0]: within a group the
    eigenvectors are not unique ("several results are correct"), only the group's projector is."""
    groups, cur = [], [0]
    for j in range(1, len(lam)):
        if abs(lam[j - 1] - lam[j]) <= rel * abs(lam[0]):
            cur.append(j)
        else:
            groups.append(cur)
            cur = [j]
    groups.append(cur)
    return groups
