"""Predict-kernel experiment on the C4 workload: fit a few trees, then time
bf_predict of the 10M-row query batch for each path/mode (CUDA events).
usage: python tools/predict_exp.py [ntree] [m]"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ipps_madougouvln16_b200 as bf  # noqa: E402
from paper_conf_ipps_madougouvln16_b200 import synthetic as S  # noqa: E402

T = int(sys.argv[1]) if len(sys.argv) > 1 else 48
m = int(sys.argv[2]) if len(sys.argv) > 2 else 10_000_000
dev = torch.device("cuda:0")
X, y, _ = S.dataset("C4")
p, n = X.shape
Xd = torch.from_numpy(X).to(dev)
yd = torch.from_numpy(y).to(dev)
g = torch.Generator(device=dev)
g.manual_seed(S.QUERY_SEED)
idx = torch.randint(0, n, (m,), device=dev, generator=g)
Qd = Xd[:, idx]
jit = torch.rand((p, m), device=dev, generator=g) < 0.5
Qd = torch.where(jit, Qd * (1.0 + 0.01 * torch.randn((p, m), device=dev, generator=g, dtype=torch.float64)), Qd).contiguous()
del idx, jit
f = bf.fit(Xd, yd, ntree=T, seed=S.FOREST_SEED + 4)
print("trees", T, "nodes", f.info.total_nodes, flush=True)
ref = None
CASES = [("node16_blk48", {"BF_PREDICT_NODE16": "1"})]
CASES += [(f"node8_blk{b}", {"BF_PREDICT_BLOCK_BYTES": str(b << 20)}) for b in (16, 24, 32, 48, 64)]
if os.environ.get("PEXP_CASES") == "env":  # one case: the caller's environment (BF_PREDICT_V, block bytes, ...)
    CASES = [("env", None)]
elif os.environ.get("PEXP_CASES"):
    CASES = [c for c in CASES if c[0] in os.environ["PEXP_CASES"].split(",")]
for name, env in CASES:
    if env is not None:
        for k in ("BF_PREDICT_NODE16", "BF_PREDICT_BLOCK_BYTES"):
            os.environ.pop(k, None)
        os.environ.update(env)
    ys, _ = f.predict(Qd, ntree_total=T)
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(3):
        ys, _ = f.predict(Qd, ntree_total=T)
    b.record()
    torch.cuda.synchronize()
    ms = a.elapsed_time(b) / 3
    bf.profile_enable(True)
    f.predict(Qd, ntree_total=T)
    torch.cuda.synchronize()
    bf.profile_enable(False)
    st = bf.profile_read()
    vis = st.get("predict_node_visits", {}).get("bytes", 0)
    fb = st.get("predict_fp64_fallbacks", {}).get("bytes", 0)
    out = ys.cpu().numpy()
    if ref is None:
        ref = out
    err = float(np.max(np.abs(out - ref) / np.abs(ref)))
    print(f"{name:22s} {ms:9.2f} ms  {m * T / ms / 1e6:8.2f} Mwalks/ms  visits/walk {vis / m / T:6.2f}  "
          f"fallback/visit {fb / max(vis, 1):.2e}  maxrel {err:.1e}", flush=True)
f.free()
