"""Print subtree-kernel phase counters (BF_SUBTREE_STATS=1) and fit times for C1/C2/C4 samples."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ["BF_SUBTREE_STATS"] = "1"
os.environ["BF_FIT_TIMING"] = "1"
import torch
import paper_conf_ipps_madougouvln16_b200 as bf
from paper_conf_ipps_madougouvln16_b200 import synthetic as S
CFGS = [("C1", 500, [0]), ("C2", 100, [0, 128]), ("C4", 16, [0, 256, 128])]
if len(sys.argv) > 1 and sys.argv[1] == "c4":
    CFGS = [("C4", 16, [0])]
for cfg, T, As in CFGS:
    X, y, c = S.dataset(cfg)
    Xd, yd = torch.from_numpy(X).cuda(), torch.from_numpy(y).cuda()
    for A in As:
        bf.fit(Xd, yd, ntree=T, seed=1, small_node_max=A).free()
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        bf.fit(Xd, yd, ntree=T, seed=1, small_node_max=A).free()
        torch.cuda.synchronize()
        print(f"{cfg} A={A} T={T}: {(time.perf_counter()-t0)*1e3:.1f} ms", file=sys.stderr, flush=True)
