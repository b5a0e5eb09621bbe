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
