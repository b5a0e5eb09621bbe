"""Measurement of the widened rows (SURVEY 8(f) NEXT-1..4) on one B200: one JSON line per row with the device
time (CUDA events, after warm-up), the dominant kernel's algorithmic GB/s against the measured HBM peak where
the row streams data, and the oracle's time on the same input where it finishes in seconds.
usage: python tools/bench_next.py > profiles/rNN/next_rows.jsonl"""
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ipps_madougouvln16_b200 as bf  # noqa: E402
from paper_conf_ipps_madougouvln16_b200 import synthetic as S  # noqa: E402
from paper_conf_ipps_madougouvln16_b200 import workflows as W  # noqa: E402

dev = torch.device("cuda:0")
try:
    HBM = float(json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"])
except Exception:
    HBM = 6650.0


def timed(fn, reps=3):
    fn()
    torch.cuda.synchronize()
    bf.profile_read()
    bf.profile_enable(True)
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(reps):
        out = fn()
    b.record()
    torch.cuda.synchronize()
    bf.profile_enable(False)
    st = bf.profile_read()
    return a.elapsed_time(b) / reps, st, out


def dominant(st, reps=3):
    k = max(st, key=lambda n: st[n]["ms"])
    d = st[k]
    gbs = d["bytes"] / (d["ms"] / 1e3) / 1e9 if d["bytes"] > 0 else None
    return {"kernel": k, "ms": d["ms"] / reps, "GBps": gbs, "frac_hbm": gbs / HBM if gbs else None}


def emit(row, **kw):
    print(json.dumps({"row": row, **kw}), flush=True)


# NEXT-1 partial dependence: C2 forest (500 trees), all 4096 training rows, 51-point grid of N
X, y, c = S.dataset("C2")
Xd, yd = torch.from_numpy(X).to(dev), torch.from_numpy(y).to(dev)
f = bf.fit(Xd, yd, ntree=500, seed=S.FOREST_SEED + 2)
m = X.shape[0] - 1
ms, st, _ = timed(lambda: f.partial_dependence(Xd, m, n_pt=51))
walks = 4096 * 51 * 500
emit("NEXT-1 partial dependence", workload="C2 forest 500 trees x 4096 rows x 51 grid points", ms=ms,
     walks_per_s=walks / (ms / 1e3), dominant=dominant(st))
f.free()

# NEXT-2 varimax of the C3 PCA loadings (k = 8)
Xc, L, M, y3 = S.gen_nw()
Xcd = torch.from_numpy(Xc).to(dev)
pc = bf.pca(Xcd, scale=True, k=8)
Ld = (pc["rotation"][:8] * pc["sdev"][:8, None]).contiguous()
ms, st, _ = timed(lambda: bf.varimax(Ld))
emit("NEXT-2 varimax", workload="C3 loadings 60 x 8", ms=ms, dominant=dominant(st))

# NEXT-3 GLM counter models: 1M runs, cubic design in log size, 64 counters
n = 1_000_000
rng = np.random.default_rng(3)
size = torch.from_numpy(32.0 * rng.integers(1, 257, n)).to(dev)
Z = W.log_size_design(size)
Yc = torch.from_numpy(rng.normal(size=(64, n))).to(dev) + torch.from_numpy(rng.normal(size=(64, 4))).to(dev) @ Z
ms, st, g = timed(lambda: bf.glm_gaussian(Z, Yc))
t0 = time.perf_counter()
np.linalg.lstsq(Z.cpu().numpy().T, Yc.cpu().numpy().T, rcond=None)
cpu_s = time.perf_counter() - t0
emit("NEXT-3 GLM counter models", workload="n=1M rows, k=4 design, r=64 counters", ms=ms,
     rows_per_s=n / (ms / 1e3), dominant=dominant(st),
     algorithmic_bytes="k_glm_cross: 8 (k + r) B per row per pass (3 passes)",
     cpu_lstsq_numpy_s=cpu_s, cpu_cores=os.cpu_count())
ms, st, _ = timed(lambda: bf.glm_predict(Z, g["coef"]))
emit("NEXT-3 GLM predict", workload="n=1M rows, k=4, r=64", ms=ms, dominant=dominant(st))

# NEXT-4 rank similarity (p = 64) and the two workflows at full config sizes
a = torch.from_numpy(rng.normal(size=64)).to(dev)
b = a + torch.from_numpy(rng.normal(size=64)).to(dev)
ms, st, _ = timed(lambda: bf.rank_similarity(a, b), reps=20)
emit("NEXT-4 rank similarity", workload="p=64", ms=ms)

size_row = X.shape[0] - 1
sizes = np.unique(X[size_row])
te_mask = np.isin(X[size_row], sizes[2::5])
tr, te = torch.from_numpy(np.nonzero(~te_mask)[0]).to(dev), torch.from_numpy(np.nonzero(te_mask)[0]).to(dev)
ms, st, r = timed(lambda: W.problem_scaling(Xd, yd, size_row, tr, te, top=6, ntree=500, seed=1), reps=1)
emit("NEXT-3 problem-scaling workflow", workload="C2 (MM), 500 trees, every 5th size unseen", ms=ms,
     keep=r["keep"], test_mse=r["test_mse"], test_explained=r["test_explained"], dominant=dominant(st, 1))
gen = torch.from_numpy(np.array([{13: 1, 15: 0, 16: 2}[int(v)] for v in M[2]])).to(dev)
ms, st, r = timed(lambda: W.hardware_scaling(Xcd, torch.from_numpy(L).to(dev), torch.from_numpy(M).to(dev),
                                             torch.from_numpy(y3).to(dev), gen, (0, 1), 2, ntree=500, seed=1), reps=1)
emit("NEXT-4 hardware-scaling workflow", workload="C3 (NW x 3 generations), 500 trees, train {0,1} test 2", ms=ms,
     k=r["k"], test_mse=r["test_mse"], test_explained=r["test_explained"],
     similarity={f"{k[0]}-{k[1]}": v for k, v in r["similarity"].items()}, dominant=dominant(st, 1))

# NEXT-3 MARS counter models (R28): one NW counter vs sequence length, 16384 runs (C3 size)
Lh = torch.from_numpy(L[None, :]).to(dev)
jc = int(np.argmax([abs(np.corrcoef(np.log2(L), c)[0, 1]) for c in Xc]))  # the counter that tracks L most
cnt = torch.from_numpy(Xc[jc]).to(dev)
ms, st, mg = timed(lambda: bf.mars_fit(Lh, cnt), reps=1)
from oracle import mars as Ms  # noqa: E402  (cpu_baseline leg: the oracle timed on the host, bounded sample)
sub = np.arange(0, L.shape[0], 8)
t0 = time.perf_counter()
Ms.mars_fit(L[None, sub], Xc[jc][sub])
cpu_s = time.perf_counter() - t0
emit("NEXT-3 MARS counter model", workload=f"C3: counter {jc} vs L, n=16384 (128 distinct L)", ms=ms,
     terms=len(mg["terms"]), rsq=mg["rsq"], dominant=dominant(st, 1),
     cpu_oracle_s_on_1_in_8_rows=cpu_s, cpu_cores=1)
