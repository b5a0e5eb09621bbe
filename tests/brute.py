"""Brute-force exact-rational tree grower (test pin for the oracle's S4).

Independent of oracle/bfo.c: written straight from PAPER.md eq.(3)
 with Python ``fractions``: for every drawn predictor j and every
split point s between two distinct values present in the node, compute

    min_c1 sum_{R1} w (y - c1)^2 + min_c2 sum_{R2} w (y - c2)^2

exactly (inner minimisers = weighted region means), pick the
minimum; ties -> lowest predictor, then lowest split value (reading R1).
No positive decrease -> leaf (reading R5).  Nodes with n_k <= nodesize are
leaves (reading R3).  Children are queued left then right (BFS ids).

The random inputs of the method (bootstrap multiplicities, the per-node
predictor subset and node keys) are passed in as callables, exactly as the
task allows for RNG-defined quantities.
"""
from __future__ import annotations

import math
from fractions import Fraction


def rss(rows, w, y):
    n = sum(w[r] for r in rows)
    s = sum(w[r] * Fraction(y[r]) for r in rows)
    mean = s / n
    return sum(w[r] * (Fraction(y[r]) - mean) ** 2 for r in rows)


def brute_tree(X, y, w, nodesize, draw=None, child_key=None):
    """X: list of p columns (lists of floats), y: list, w: multiplicities.
    draw(key) -> iterable of features; child_key(key, side) -> key.
    Returns list of nodes in BFS order: dict(feature, a, b, left, count, value, drss)."""
    p = len(X)
    n = len(y)
    rows0 = [i for i in range(n) if w[i] > 0]
    queue = [(rows0, 0)]
    nodes = [None]
    ids = [0]
    head = 0
    while head < len(queue):
        rows, key = queue[head]
        nid = ids[head]
        head += 1
        nk = sum(w[r] for r in rows)
        value = sum(w[r] * Fraction(y[r]) for r in rows) / nk
        node = dict(feature=-1, a=None, b=None, left=-1, count=nk, value=value, drss=Fraction(0))
        nodes[nid] = node
        if nk <= nodesize:
            continue
        feats = range(p) if draw is None else sorted(set(int(f) for f in draw(key)))
        parent = rss(rows, w, y)
        best = None
        for f in feats:
            vals = sorted(set(X[f][r] for r in rows))
            for a, b in zip(vals, vals[1:]):
                L = [r for r in rows if X[f][r] <= a]
                R = [r for r in rows if X[f][r] > a]
                tot = rss(L, w, y) + rss(R, w, y)
                cand = (tot, f, a, b, L, R)
                if best is None or (tot, f, a) < (best[0], best[1], best[2]):
                    best = cand
        if best is None or best[0] == parent:
            continue
        tot, f, a, b, L, R = best
        node.update(feature=f, a=a, b=b, drss=parent - tot)
        lid = len(nodes)
        nodes.extend([None, None])
        node["left"] = lid
        kl = child_key(key, 0) if child_key else 0
        kr = child_key(key, 1) if child_key else 0
        queue.append((L, kl))
        ids.append(lid)
        queue.append((R, kr))
        ids.append(lid + 1)
    return nodes


def brute_walk(nodes, x):
    """Leaf value (exact Fraction) of one brute tree for the row x (list of p values):
    x_f <= s -> left, else right (eq.(2)) with s the midpoint (a + b)/2 of the
    gap the split falls in (reading R2).  Rows outside the node's in-bag sample (OOB rows,
    permuted values) can fall strictly inside (a, b), so s matters there."""
    k = 0
    while nodes[k]["feature"] >= 0:
        nd = nodes[k]
        s = (Fraction(nd["a"]) + Fraction(nd["b"])) / 2
        k = nd["left"] if Fraction(x[nd["feature"]]) <= s else nd["left"] + 1
    return nodes[k]["value"]


def brute_importance(X, y, trees, ws, perms):
    """Exact-rational OOB permutation importance, written from P:130 ("increase in
    prediction error when the values of a predictor in the OOB sample are permuted")
    and the OOB error of P:157, for a forest given as brute trees.

    X: list of p columns, y: list, trees[t]: brute_tree nodes, ws[t]: multiplicities,
    perms[t][m]: the permutation of [0, n_o) applied to tree t's OOB rows for predictor m
    (an RNG-defined input).  Every quantity is an exact Fraction:
      O_t   = OOB rows ascending, n_o = |O_t|
      e_t   = sum_a (y - f_t(x_{O_t[a]}))^2
      e_tm  = sum_a (y - f_t(x~_a))^2,  x~_a = x_{O_t[a]} with column m := x_{O_t[pi(a)], m}
      d_tm  = (e_tm - e_t) / n_o          (0 when n_o = 0, reading R13)
    and the aggregation over T trees: raw_m = mean_t d_tm, var_m = mean_t d_tm^2 - raw_m^2
    (R's one-pass importanceSD form; equal in exact arithmetic to the two-pass form),
    sd_m = sqrt(var_m / T).  OOB: yhat_i = mean over trees with w_t[i] = 0 of f_t(x_i);
    oob_mse = mean over rows with >= 1 OOB tree of (y_i - yhat_i)^2; rsq = 1 - oob_mse / var_pop(y).
    """
    p, n, T = len(X), len(y), len(trees)
    row = lambda i: [X[j][i] for j in range(p)]
    d = [[Fraction(0)] * p for _ in range(T)]
    e = [Fraction(0)] * T
    nout = [0] * T
    osum = [Fraction(0)] * n
    ocnt = [0] * n
    for t in range(T):
        O = [i for i in range(n) if ws[t][i] == 0]
        no = len(O)
        nout[t] = no
        et = Fraction(0)
        for i in O:
            f = brute_walk(trees[t], row(i))
            osum[i] += f
            ocnt[i] += 1
            et += (Fraction(y[i]) - f) ** 2
        e[t] = et
        if no == 0:
            continue
        for m in range(p):
            pi = perms[t][m]
            etm = Fraction(0)
            for a, i in enumerate(O):
                x = row(i)
                x[m] = X[m][O[pi[a]]]
                etm += (Fraction(y[i]) - brute_walk(trees[t], x)) ** 2
            d[t][m] = (etm - et) / no
    raw = [sum(d[t][m] for t in range(T)) / T for m in range(p)]
    var = [sum(d[t][m] ** 2 for t in range(T)) / T - raw[m] ** 2 for m in range(p)]
    sd = [math.sqrt(v / T) for v in var]
    rows = [i for i in range(n) if ocnt[i] > 0]
    mse = sum((Fraction(y[i]) - osum[i] / ocnt[i]) ** 2 for i in rows) / len(rows) if rows else Fraction(0)
    ybar = sum(Fraction(v) for v in y) / n
    varp = sum((Fraction(v) - ybar) ** 2 for v in y) / n
    return dict(d=d, e=e, nout=nout, osum=osum, ocnt=ocnt, raw=raw, var=var, sd=sd, oob_mse=mse,
                rsq=(1 - mse / varp) if varp else Fraction(0))
