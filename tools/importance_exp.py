"""bf_oob_importance timing on C4 (T trees): Node16 vs compact-node walks, per-kernel device times."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import paper_conf_ipps_madougouvln16_b200 as bf
from paper_conf_ipps_madougouvln16_b200 import synthetic as S
T = int(sys.argv[1]) if len(sys.argv) > 1 else 40
X, y, c = S.dataset("C4")
Xd, yd = torch.from_numpy(X).cuda(), torch.from_numpy(y).cuda()
f = bf.fit(Xd, yd, ntree=T, seed=S.FOREST_SEED + 4)
ref = None
for name, env in [("node16", {"BF_PREDICT_NODE16": "1"}), ("node8", {})]:
    os.environ.pop("BF_PREDICT_NODE16", None)
    os.environ.update(env)
    f.oob_importance(Xd, yd)
    torch.cuda.synchronize()
    bf.profile_enable(True)
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    r = f.oob_importance(Xd, yd)
    b.record()
    torch.cuda.synchronize()
    bf.profile_enable(False)
    st = bf.profile_read()
    top = sorted(st.items(), key=lambda kv: -kv[1]["ms"])[:5]
    d = r["d_slots"].cpu().numpy()
    if ref is None:
        ref = d
    err = float(np.max(np.abs(d - ref)) / np.abs(ref).max())
    print(f"{name}: {a.elapsed_time(b):.1f} ms  " + " ".join(f"{k}={v['ms']:.1f}" for k, v in top) + f"  maxdiff/max {err:.1e}", flush=True)
f.free()
