"""Tree-parallel multi-GPU layer.

Trees are independent units ("for each of those samples, grow an
unpruned regression tree"), so the forest shards by tree: rank r of R grows
global trees [floor(rT/R), floor((r+1)T/R)).  Every random stream is keyed by
the GLOBAL tree id (S3), so the forest is bit-identical for any R.
The data path has no collective; the exchanges are:

  * prediction: each rank sums its own trees' leaf values, then one
    all-reduce(sum) of the m partial sums (PAPER.md:95 step 3);
  * importance: per-tree slots (T x p) are disjoint between ranks, so an
    all-reduce(sum) of zero-padded slots is an exact all-gather; OOB row sums
    and counts are all-reduced (S6-S8);
  * forest gather (export / full-forest predict on every rank): all-gather of
    per-rank node counts, then a padded all-gather of the node arrays.

All functions take torch.distributed process groups and work with NCCL (CUDA
tensors) or gloo (CPU tensors: the world-size-2 tests).
"""
from __future__ import annotations

import numpy as np
import torch
import torch.distributed as dist

ARRAYS = ("feature", "left", "thr_or_value", "count", "value", "drss")


def tree_range(rank: int, world: int, ntree: int) -> tuple[int, int]:
    return (rank * ntree) // world, ((rank + 1) * ntree) // world


def _dev(group) -> torch.device:
    backend = dist.get_backend(group)
    return torch.device("cuda", torch.cuda.current_device()) if backend == "nccl" else torch.device("cpu")


def _all_gather_var(t: torch.Tensor, group) -> list[torch.Tensor]:
    """All-gather of 1-D tensors of different lengths (pad to the max, trim)."""
    world = dist.get_world_size(group)
    n = torch.tensor([t.numel()], dtype=torch.int64, device=t.device)
    ns = [torch.zeros_like(n) for _ in range(world)]
    dist.all_gather(ns, n, group=group)
    ns = [int(x.item()) for x in ns]
    mx = max(ns) if ns else 0
    pad = torch.zeros(mx, dtype=t.dtype, device=t.device)
    pad[: t.numel()] = t
    outs = [torch.empty_like(pad) for _ in range(world)]
    dist.all_gather(outs, pad, group=group)
    return [o[:k] for o, k in zip(outs, ns)]


def gather_forest_arrays(local: dict, group=None) -> dict:
    """local: exported arrays of this rank's trees (Forest.export() format:
    tree_off (nt+1), feature, left, thr_or_value, count, value, drss).
    Returns the same arrays for ALL trees in global tree order (rank order)."""
    dev = _dev(group)
    off = np.asarray(local["tree_off"], np.int64)
    sizes = torch.from_numpy(np.diff(off)).to(dev)
    all_sizes = torch.cat(_all_gather_var(sizes, group)).cpu().numpy()
    out = {"tree_off": np.concatenate([[0], np.cumsum(all_sizes)]).astype(np.int64)}
    for k in ARRAYS:
        a = torch.from_numpy(np.ascontiguousarray(local[k])).to(dev)
        out[k] = torch.cat(_all_gather_var(a, group)).cpu().numpy()
    return out


def merge_importance(acc: dict, tree_begin: int, tree_end: int, ntree: int, group=None) -> dict:
    """Place this rank's per-tree slots at their global rows and all-reduce.
    Disjoint slots -> the sum is an exact all-gather (bit-identical to one
    process).  oob_sum / oob_cnt are summed across ranks."""
    dev = _dev(group)
    p = acc["d_slots"].shape[1]
    out = {}
    for k in ("d_slots", "npur_slots"):
        g = torch.zeros((ntree, p), dtype=torch.float64, device=dev)
        g[tree_begin:tree_end] = torch.as_tensor(np.asarray(acc[k]) if isinstance(acc[k], np.ndarray) else acc[k]).to(dev)
        dist.all_reduce(g, group=group)
        out[k] = g
    for k, dt in (("e_t", torch.float64), ("nout_t", torch.int64)):
        g = torch.zeros(ntree, dtype=dt, device=dev)
        v = torch.as_tensor(np.asarray(acc[k]) if isinstance(acc[k], np.ndarray) else acc[k]).to(dev)
        g[tree_begin:tree_end] = v[: tree_end - tree_begin].to(dt)
        dist.all_reduce(g, group=group)
        out[k] = g
    for k in ("oob_sum", "oob_cnt"):
        v = torch.as_tensor(np.asarray(acc[k]) if isinstance(acc[k], np.ndarray) else acc[k]).to(dev).clone()
        dist.all_reduce(v, group=group)
        out[k] = v
    return out


def allreduce_predictions(yhat_sum: torch.Tensor, ntree: int, group=None) -> torch.Tensor:
    """Sum the ranks' partial tree sums and average over the whole forest."""
    y = yhat_sum.clone()
    dist.all_reduce(y, group=group)
    return y / ntree


def fit_sharded(X, y, ntree: int, group=None, **kw):
    """Grow this rank's share of a T-tree forest through the C ABI (bf_fit)."""
    from . import fit
    rank, world = dist.get_rank(group), dist.get_world_size(group)
    lo, hi = tree_range(rank, world, ntree)
    return fit(X, y, ntree=ntree, tree_begin=lo, tree_end=hi, **kw), (lo, hi)
