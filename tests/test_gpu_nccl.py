"""Multi-GPU tree-parallel layer over NCCL: needs >= 2 visible GPUs and is
skipped otherwise (the single-GPU gpurun boxes).  Two ranks grow their tree ranges through the C ABI (bf_fit
with tree_begin / tree_end), merge the importance slots and OOB sums with NCCL all-reduces, all-reduce the
prediction partial sums and gather the forests; rank 0 compares with one process holding every tree: forests
and importance slots exactly (disjoint slots, global-tree-id keyed RNG), predictions and OOB sums to rounding.
The same exchanges run on gloo in tests/test_distributed.py."""
from __future__ import annotations

import os
import socket

import numpy as np
import pytest

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available() or torch.cuda.device_count() < 2:
    pytest.skip("needs >= 2 CUDA devices", allow_module_level=True)

import torch.distributed as dist  # noqa: E402
import torch.multiprocessing as mp  # noqa: E402

T = 12


def _port() -> int:
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    torch.cuda.set_device(rank)
    dist.init_process_group("nccl", rank=rank, world_size=world, device_id=torch.device("cuda", rank))
    try:
        import paper_conf_ipps_madougouvln16_b200 as bf
        from paper_conf_ipps_madougouvln16_b200 import distributed as D
        from paper_conf_ipps_madougouvln16_b200 import synthetic as S
        dev = torch.device("cuda", rank)
        X, y = S.gen_mm(n=2048)
        Xd, yd = torch.from_numpy(X).to(dev), torch.from_numpy(y).to(dev)
        f, (lo, hi) = D.fit_sharded(Xd, yd, T, seed=S.FOREST_SEED + 11)
        acc = f.oob_importance(Xd, yd)
        merged = D.merge_importance(acc, lo, hi, T)
        Q = torch.from_numpy(S.gen_query(X, 999)).to(dev)
        ps, _ = f.predict(Q, ntree_total=T)
        pred = D.allreduce_predictions(ps, T)
        gathered = D.gather_forest_arrays(f.export())
        if rank == 0:
            full = bf.fit(Xd, yd, ntree=T, seed=S.FOREST_SEED + 11)
            ref = {k: v.cpu().numpy() for k, v in full.oob_importance(Xd, yd).items()}
            e = full.export()
            _, yr = full.predict(Q, ntree_total=T)
            ok = {
                "d_slots": np.array_equal(merged["d_slots"].cpu().numpy(), ref["d_slots"]),
                "npur": np.array_equal(merged["npur_slots"].cpu().numpy(), ref["npur_slots"]),
                "nout": np.array_equal(merged["nout_t"].cpu().numpy(), ref["nout_t"]),
                "oob_cnt": np.array_equal(merged["oob_cnt"].cpu().numpy(), ref["oob_cnt"]),
                "oob_sum": bool(np.allclose(merged["oob_sum"].cpu().numpy(), ref["oob_sum"], rtol=1e-12, atol=0)),
                "pred": bool(torch.allclose(pred, yr, rtol=1e-12, atol=0)),
                "forest_sizes": np.array_equal(np.diff(gathered["tree_off"]), np.diff(e["tree_off"])),
                "nccl": dist.get_backend() == "nccl" and dist.get_world_size() == world,
            }
            q.put(ok)
    finally:
        dist.destroy_process_group()


def test_nccl_world2_merge_equals_single_process():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    ok = q.get(timeout=600)
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    assert all(ok.values()), ok
