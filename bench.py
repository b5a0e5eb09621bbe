#!/usr/bin/env python
"""bench.py -- BlackForest hot path on B200: trees/s (fit) and predictions/s.

One step = one pass of the whole hot path over the
configured workload:
    bf_fit (this rank's share of the T trees, presort included)
  + bf_predict of the query batch (C5: 10M rows) with this rank's trees,
    partial sums all-reduced over ranks (NCCL)
  + bf_oob_importance of this rank's trees, disjoint slots all-reduced,
    bf_importance_finalize
  + bf_pca of the training counters.
value = T / step time (whole-job trees/s, all ranks); predictions/s are
reported beside it.  Inputs are resident in HBM before the timed region;
`e2e` repeats the step through the C ABI with HOST (pinned) buffers.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]
                  [--config C4] [--ntree T] [--m-query M]
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

MEASURED = os.path.join(ROOT, "MEASURED_PEAKS.json")
FALLBACK_HBM_GBS = 6650.0  # B200_PROFILING.md fallback


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=3)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default="C4")
    ap.add_argument("--ntree", type=int, default=0, help="override T (default: the config's)")
    ap.add_argument("--m-query", type=int, default=-1, help="override the query batch (default: the config's)")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--e2e-steps", type=int, default=1)
    return ap.parse_args()


def peaks():
    try:
        d = json.load(open(MEASURED))
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    except Exception:
        return FALLBACK_HBM_GBS, "fallback (B200_PROFILING.md)"


def ncu_traffic(kernel: str):
    """DRAM bytes (read + write) per launch of `kernel` from the newest committed
    `ncu --set full` summary under profiles/ (tools/ncu_summary.py), or None."""
    import glob
    for d in sorted(glob.glob(os.path.join(ROOT, "profiles", "r[0-9]*")), reverse=True):
        f = os.path.join(d, f"full_{kernel}.json")
        if os.path.exists(f):
            try:
                return float(json.load(open(f))["dram_bytes"]), os.path.relpath(f, ROOT)
            except Exception:
                pass
    return None, None


def ncu_issue(kernel: str):
    """Issue-slot utilisation of `kernel` from the newest committed ncu summary: the bound of the latency /
    issue-limited kernels (4 warp-instructions per SM per cycle is the sm_100 issue peak)."""
    import glob
    for d in sorted(glob.glob(os.path.join(ROOT, "profiles", "r[0-9]*")), reverse=True):
        f = os.path.join(d, f"full_{kernel}.json")
        if os.path.exists(f):
            try:
                m = json.load(open(f))["metrics"]
                ipc = float(m["sm__inst_executed.avg.per_cycle_active"])
                return {"bound": "issue", "achieved_ipc": ipc, "peak_ipc": 4.0, "frac": ipc / 4.0,
                        "warps_active_pct": float(m["sm__warps_active.avg.pct_of_peak_sustained_active"]),
                        "dram_pct_of_peak": float(m["gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed"]),
                        "source": os.path.relpath(f, ROOT)}
            except Exception:
                pass
    return None


class Clocks:
    """nvidia-smi sampling during the timed region (B200_PROFILING.md clocks line)."""

    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.index = index
        self.rows = []
        self._stop = threading.Event()
        self._t = None

    def _run(self):
        try:
            p = subprocess.Popen(["nvidia-smi", f"--id={self.index}", f"--query-gpu={self.Q}",
                                  "--format=csv,noheader,nounits", "-lms", "200"],
                                 stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
        except Exception:
            return
        try:
            while not self._stop.is_set():
                line = p.stdout.readline()
                if not line:
                    break
                self.rows.append([x.strip() for x in line.split(",")])
        finally:
            p.terminate()

    def __enter__(self):
        self._t = threading.Thread(target=self._run, daemon=True)
        self._t.start()
        return self

    def __exit__(self, *a):
        self._stop.set()
        if self._t:
            self._t.join(timeout=3)

    def summary(self):
        if not self.rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        sm = [float(r[1]) for r in self.rows if len(r) > 2 and r[1].replace(".", "").isdigit()]
        mx = [float(r[2]) for r in self.rows if len(r) > 2 and r[2].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = set()
        for r in self.rows:
            for k, nm in enumerate(names):
                if len(r) > 5 + k and r[5 + k].lower() == "active":
                    reasons.add(nm)
        return {"sm_mhz": float(np.median(sm)) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": sorted(reasons), "samples": len(self.rows)}


def dist_setup(args):
    import torch
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if args.impl == "ours":
        torch.cuda.set_device(local)
    if world > 1:
        import torch.distributed as dist
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        dist.init_process_group("nccl" if args.impl == "ours" else "gloo")
    return rank, world, local


def workload(args):
    from paper_conf_ipps_madougouvln16_b200 import synthetic as S
    cfg = S.CONFIGS[args.config]
    T = args.ntree or cfg.ntree
    m = cfg.m_query if args.m_query < 0 else args.m_query
    return S, cfg, T, m


# ---------------------------------------------------------------------------- reference arm (CPU oracle)
def run_reference(args):
    rank, world, _ = dist_setup(args)
    if rank != 0:
        return
    from oracle import oracle as O
    S, cfg, T, m = workload(args)
    X, y, _ = S.dataset(args.config)
    cores = os.cpu_count() or 1
    k = cores  # one tree per host thread per step: the bounded sample
    times = []
    for it in range(args.warmup + args.steps):
        t0 = time.perf_counter()
        O.fit(X, y, ntree=T, seed=S.FOREST_SEED + 4, tree_begin=(it * k) % T, tree_end=min(T, (it * k) % T + k),
              nthreads=cores)
        times.append(time.perf_counter() - t0)
    dt = float(np.mean(times[args.warmup:]))
    val = k / dt
    print(json.dumps({
        "impl": "reference", "metric": "trees/sec fit", "value": val, "unit": "trees/s", "n_gpus": args.gpus,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": dt * 1e3, "higher_is_better": True,
        "scaling": "strong", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": {"workload": cfg.name, "n": cfg.n, "p": cfg.p, "ntree": T, "mtry": cfg.mtry or max(cfg.p // 3, 1),
                   "nodesize": cfg.nodesize},
        "cpu_baseline": {"value": val, "unit": "trees/s", "cores": cores, "kind": "oracle",
                         "sample": f"{k} trees of {cfg.name} per step grown by oracle bfo_fit, one per host thread "
                                   f"(fit only: predict/importance of the CPU oracle would take minutes per tree)"},
        "e2e": {"value": val, "unit": "trees/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }))


# ---------------------------------------------------------------------------- our arm
def run_ours(args):
    import torch
    import torch.distributed as dist

    import paper_conf_ipps_madougouvln16_b200 as bf
    from paper_conf_ipps_madougouvln16_b200 import distributed as D

    rank, world, local = dist_setup(args)
    dev = torch.device("cuda", local)
    S, cfg, T, m = workload(args)
    t0, t1 = D.tree_range(rank, world, T)
    X, y, _ = S.dataset(args.config)
    p, n = X.shape
    Xh = torch.from_numpy(X).pin_memory()
    yh = torch.from_numpy(y).pin_memory()
    Xd = Xh.to(dev)
    yd = yh.to(dev)
    # query batch: drawn on the device from the training rows (seeded; synthetic-input plumbing only)
    g = torch.Generator(device=dev)
    g.manual_seed(S.QUERY_SEED)
    Qd = None
    if m > 0:
        idx = torch.randint(0, n, (m,), device=dev, generator=g)
        Qd = Xd[:, idx]
        jit = torch.rand((p, m), device=dev, generator=g) < 0.5
        Qd = torch.where(jit, Qd * (1.0 + 0.01 * torch.randn((p, m), device=dev, generator=g, dtype=torch.float64)), Qd)
        Qd = Qd.contiguous()
        del idx, jit
    k_pca = 8
    stream = torch.cuda.current_stream()
    ev = lambda: torch.cuda.Event(enable_timing=True)

    def step(Xs, ys_, Qs, host: bool):
        """One pass of the hot path; returns per-phase events and the result scalars."""
        e = [ev() for _ in range(5)]
        e[0].record(stream)
        forest = bf.fit(Xs, ys_, ntree=T, seed=S.FOREST_SEED + 4, tree_begin=t0, tree_end=t1)
        e[1].record(stream)
        pred = None
        if Qs is not None:
            ps, _ = forest.predict(Qs, ntree_total=T)
            if host:
                ps = torch.from_numpy(ps).to(dev)
            pred = D.allreduce_predictions(ps, T) if world > 1 else ps / T
        e[2].record(stream)
        acc = forest.oob_importance(Xs, ys_)
        if host:
            acc = {k: torch.from_numpy(v).to(dev) for k, v in acc.items()}
        if world > 1:  # disjoint per-tree slots: the all-reduce is an exact all-gather
            m = D.merge_importance(acc, t0, t1, T)
            dsl, npu, osum, ocnt = m["d_slots"], m["npur_slots"], m["oob_sum"], m["oob_cnt"]
        else:
            dsl, npu, osum, ocnt = acc["d_slots"], acc["npur_slots"], acc["oob_sum"], acc["oob_cnt"]
        fin = bf.importance_finalize(dsl, npu, osum, ocnt, yd)
        e[3].record(stream)
        pc = bf.pca(Xs, scale=True, k=k_pca)
        e[4].record(stream)
        res = fin["oob_mse"]
        if host:
            out = res.cpu()  # device -> host read of the step's result
            if pred is not None:
                pred.cpu()
        forest.free()
        return e, res, pc

    def barrier():
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()

    # warm-up
    for _ in range(args.warmup):
        step(Xd, yd, Qd, False)
    barrier()
    # timed region (device-resident inputs); L2 note: X (p*n*8 B) and the lists exceed L2
    L0 = bf.launch_count()
    bf.profile_enable(True)
    phase = np.zeros(4)
    with Clocks(local) as clk:
        barrier()
        start, end = ev(), ev()
        start.record(stream)
        for _ in range(args.steps):
            e, res, _ = step(Xd, yd, Qd, False)
            torch.cuda.synchronize()
            phase += [e[i].elapsed_time(e[i + 1]) for i in range(4)]
        end.record(stream)
        barrier()
    bf.profile_enable(False)
    launches = (bf.launch_count() - L0) // args.steps
    stats = bf.profile_read()
    ms = start.elapsed_time(end) / args.steps
    msmax = torch.tensor([ms], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(msmax, op=dist.ReduceOp.MAX)
    ms = float(msmax.item())
    phase /= args.steps

    # e2e through the C ABI with host (pinned) buffers
    e2e = None
    if not args.no_e2e:
        Qh = Qd.cpu().pin_memory() if Qd is not None else None
        Xn, yn = Xh.numpy(), yh.numpy()
        Qn = Qh.numpy() if Qh is not None else None
        barrier()
        s2, e2 = ev(), ev()
        s2.record(stream)
        for _ in range(args.e2e_steps):
            step(Xn, yn, Qn, True)
        e2.record(stream)
        barrier()
        me = torch.tensor([s2.elapsed_time(e2) / args.e2e_steps], dtype=torch.float64, device=dev)
        if world > 1:
            dist.all_reduce(me, op=dist.ReduceOp.MAX)
        # X is staged by bf_fit, bf_oob_importance and bf_pca; y by fit and importance
        h2d = (3 * X.nbytes + 2 * y.nbytes + (Qn.nbytes if Qn is not None else 0))
        e2e = {"value": T / (float(me.item()) / 1e3), "unit": "trees/s", "h2d_bytes_per_step": int(h2d),
               "d2h_bytes_per_step": int(8 * m + 8 + 2 * 8 * (t1 - t0) * p + 12 * n + 16 * (t1 - t0) + 8 * p * (p + 1) + 8 * n * k_pca),
               "ms_per_step": float(me.item())}

    if rank != 0:
        return
    # roofline of the dominant kernel (by device time in the timed region)
    hbm, hbm_src = peaks()
    kern = {k: v for k, v in stats.items() if v["ms"] > 0}
    dom = max(kern, key=lambda k: kern[k]["ms"]) if kern else None
    roof = None
    if dom:
        d = kern[dom]
        achieved = d["bytes"] / (d["ms"] / 1e3) / 1e9 if d["bytes"] > 0 else 0.0
        traffic, tsrc = ncu_traffic(dom)
        roof = {"kernel": dom, "bound": "hbm", "achieved": achieved, "peak": hbm, "unit": "GB/s",
                "frac": achieved / hbm, "traffic": traffic, "traffic_source": tsrc, "peak_source": hbm_src,
                "algorithmic_bytes_per_launch": d["bytes"] / max(d["launches"], 1),
                "share_of_step": d["ms"] / args.steps / ms,
                "avg_launch_ms": d["ms"] / max(d["launches"], 1),
                "issue": ncu_issue(dom)}
    kernels = {k: {"ms_per_step": v["ms"] / args.steps, "launches_per_step": v["launches"] / args.steps,
                   "GBps": (v["bytes"] / (v["ms"] / 1e3) / 1e9) if v["ms"] > 0 and v["bytes"] > 0 else None,
                   "frac_hbm": (v["bytes"] / (v["ms"] / 1e3) / 1e9 / hbm) if v["ms"] > 0 and v["bytes"] > 0 else None}
               for k, v in sorted(stats.items(), key=lambda kv: -kv[1]["ms"]) if v["launches"] > 0}
    vis = stats.get("predict_node_visits", {}).get("bytes", 0.0)
    fbk = stats.get("predict_fp64_fallbacks", {}).get("bytes", 0.0)
    cpu = None
    if not args.no_cpu_baseline and world == 1:
        cpu = cpu_baseline(args, S, cfg, T, X, y)
    out = {
        "metric": "trees/sec fit (whole hot-path step) and predictions/sec",
        "value": T / (ms / 1e3), "unit": "trees/s", "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": ms, "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "f64",
        "data": "synthetic",
        "config": {"workload": cfg.name, "n": n, "p": p, "ntree": T, "mtry": max(p // 3, 1), "nodesize": cfg.nodesize,
                   "m_query": m, "pca_k": k_pca, "parallelism": f"tree-sharded x{world}",
                   "l2": "inputs larger than L2 (X 512 MB, lists GBs); no flush"},
        "predictions_per_s": (m / (phase[1] / 1e3)) if m and phase[1] > 0 else None,
        "predict_node_visits_per_walk": (vis / args.steps / (m * (t1 - t0))) if m and vis else None,
        "predict_fp64_fallbacks_per_visit": (fbk / vis) if vis else None,
        "phases_ms": {"fit": phase[0], "predict": phase[1], "importance": phase[2], "pca": phase[3]},
        "gpu_launches": int(launches),
        "roofline": roof,
        "kernels": kernels,
        "clocks": clk.summary(),
        "e2e": e2e,
        "cpu_baseline": cpu,
    }
    print(json.dumps(out))


def cpu_baseline(args, S, cfg, T, X, y):
    """The oracle as it stands, on the host cores, on a bounded sample: one
    C4 tree per host thread (fit only)."""
    from oracle import oracle as O
    cores = os.cpu_count() or 1
    k = cores
    t0 = time.perf_counter()
    O.fit(X, y, ntree=T, seed=S.FOREST_SEED + 4, tree_begin=0, tree_end=min(k, T), nthreads=cores)
    dt = time.perf_counter() - t0
    return {"value": min(k, T) / dt, "unit": "trees/s", "cores": cores, "kind": "oracle",
            "sample": f"{min(k, T)} trees of {cfg.name} grown by oracle bfo_fit, one per host thread, "
                      f"{dt:.1f} s (fit only; predict/importance excluded)"}


def main():
    args = parse()
    if args.impl == "reference":
        run_reference(args)
    else:
        run_ours(args)
    if int(os.environ.get("WORLD_SIZE", "1")) > 1:
        import torch.distributed as dist
        if dist.is_initialized():
            dist.destroy_process_group()


if __name__ == "__main__":
    main()
