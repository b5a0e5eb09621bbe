"""Multi-process (gloo, world size 2, CPU) tests of the tree-parallel layer
(paper_conf_ipps_madougouvln16_b200/distributed.py).

Each rank grows its tree range with the CPU oracle (the product's exchanges
are what is tested here: the CUDA path is exercised by the -m gpu tests) and
the merged results must equal one process holding every tree: importance
slots and OOB counts exactly (disjoint slots: the all-reduce is an
all-gather), OOB sums and predictions to rounding, gathered forests exactly.
"""
from __future__ import annotations

import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

T = 10


def _free_port() -> int:
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _tree_arrays(of, nt):
    """Forest.export()-style arrays of an oracle forest's local trees."""
    trees = [of.tree(i) for i in range(nt)]
    cat = lambda xs, dt: np.concatenate(xs).astype(dt) if xs else np.zeros(0, dt)
    out = {"tree_off": np.concatenate([[0], np.cumsum([t["feature"].size for t in trees])]).astype(np.int64)}
    out["feature"] = cat([t["feature"] for t in trees], np.int32)
    out["left"] = cat([t["left"] for t in trees], np.int32)
    out["thr_or_value"] = cat([np.where(t["feature"] >= 0, t["thr"], t["value"]) for t in trees], np.float64)
    out["count"] = cat([t["count"] for t in trees], np.int32)
    out["value"] = cat([t["value"] for t in trees], np.float64)
    out["drss"] = cat([t["drss"] for t in trees], np.float64)
    return out


def _worker(rank, world, port, q, T=T):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from oracle import oracle as O
        from paper_conf_ipps_madougouvln16_b200 import distributed as D
        from paper_conf_ipps_madougouvln16_b200 import synthetic as S
        X, y = S.gen_reduction()
        seed = S.FOREST_SEED + 9
        lo, hi = D.tree_range(rank, world, T)
        of = O.fit(X, y, ntree=T, seed=seed, tree_begin=lo, tree_end=hi)
        acc = of.oob_importance(X, y)
        merged = D.merge_importance(acc, lo, hi, T)
        Q = S.gen_query(X, 333)
        pred = D.allreduce_predictions(torch.from_numpy(of.predict_sum(Q)), T)
        gathered = D.gather_forest_arrays(_tree_arrays(of, hi - lo))
        if rank == 0:
            full = O.fit(X, y, ntree=T, seed=seed)
            ref = full.oob_importance(X, y)
            ok = {
                "d_slots": np.array_equal(merged["d_slots"].numpy(), ref["d_slots"]),
                "npur": np.array_equal(merged["npur_slots"].numpy(), ref["npur_slots"]),
                "e_t": np.array_equal(merged["e_t"].numpy(), ref["e_t"]),
                "nout": np.array_equal(merged["nout_t"].numpy(), ref["nout_t"]),
                "oob_cnt": np.array_equal(merged["oob_cnt"].numpy(), ref["oob_cnt"]),
                "oob_sum": bool(np.allclose(merged["oob_sum"].numpy(), ref["oob_sum"], rtol=1e-12, atol=0)),
                "pred": bool(np.allclose(pred.numpy(), full.predict_sum(Q) / T, rtol=1e-12, atol=0)),
            }
            fa = _tree_arrays(full, T)
            ok["forest"] = all(np.array_equal(gathered[k], fa[k]) for k in fa)
            q.put(ok)
    finally:
        dist.destroy_process_group()


def test_tree_range_partitions_the_forest():
    from paper_conf_ipps_madougouvln16_b200 import distributed as D
    for world in (1, 2, 3, 8):
        for ntree in (1, 7, 500, 1000):
            r = [D.tree_range(k, world, ntree) for k in range(world)]
            assert r[0][0] == 0 and r[-1][1] == ntree
            assert all(r[k][1] == r[k + 1][0] for k in range(world - 1))
            assert all(hi - lo in (ntree // world, ntree // world + 1) for lo, hi in r)


@pytest.mark.parametrize("ntree", [T, 1])
def test_gloo_world2_merge_equals_single_process(ntree):
    """ntree = 1 < world: rank 0 owns the empty range [0, 0) and contributes exact zeros."""
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q, ntree)) for r in range(2)]
    for p in procs:
        p.start()
    ok = q.get(timeout=120)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    assert all(ok.values()), ok
