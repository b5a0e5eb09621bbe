"""Fit time of C4 (T trees) for several subtree capacities A, with the fit phase timer and subtree counters."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ["BF_FIT_TIMING"] = "1"
if len(sys.argv) > 2 and sys.argv[2] == "stats":
    os.environ["BF_SUBTREE_STATS"] = "1"
import torch
import paper_conf_ipps_madougouvln16_b200 as bf
from paper_conf_ipps_madougouvln16_b200 import synthetic as S
T = int(sys.argv[1]) if len(sys.argv) > 1 else 40
X, y, c = S.dataset("C4")
Xd, yd = torch.from_numpy(X).cuda(), torch.from_numpy(y).cuda()
for A in [int(a) for a in os.environ.get("AS", "0,384,256,192").split(",")]:
    bf.fit(Xd, yd, ntree=T, seed=1, small_node_max=A).free()
    torch.cuda.synchronize()
    bf.profile_enable(True)
    t0 = time.perf_counter()
    bf.fit(Xd, yd, ntree=T, seed=1, small_node_max=A).free()
    torch.cuda.synchronize()
    dt = time.perf_counter() - t0
    bf.profile_enable(False)
    st = bf.profile_read()
    top = sorted(st.items(), key=lambda kv: -kv[1]["ms"])[:6]
    print(f"A={A} T={T}: {dt*1e3:.1f} ms  " + " ".join(f"{k}={v['ms']:.0f}" for k, v in top), flush=True)
