"""Small end-to-end workload for compute-sanitizer (memcheck / racecheck / synccheck): a C1-sized fit with both
phases (small subtree capacity so the global phase runs too), predict (both node formats), OOB importance,
PCA, varimax, GLM, MARS and rank similarity."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ipps_madougouvln16_b200 as bf  # noqa: E402
from paper_conf_ipps_madougouvln16_b200 import synthetic as S  # noqa: E402

dev = torch.device("cuda:0")
X, y = S.gen_reduction()
Xd, yd = torch.from_numpy(X).to(dev), torch.from_numpy(y).to(dev)
for A in (0, 16):
    f = bf.fit(Xd, yd, ntree=6, seed=3, small_node_max=A, trees_in_flight=3)
    f.predict(Xd, ntree_total=6)
    os.environ["BF_PREDICT_NODE16"] = "1"
    f.predict(Xd, ntree_total=6)
    os.environ.pop("BF_PREDICT_NODE16")
    f.oob_importance(Xd, yd)
    f.partial_dependence(Xd, 3, n_pt=5)
    f.free()
pc = bf.pca(Xd, scale=True, k=4)
bf.varimax((pc["rotation"][:4] * pc["sdev"][:4, None]).contiguous())
Z = torch.stack([torch.ones(256, dtype=torch.float64, device=dev), Xd[0]])
bf.glm_gaussian(Z, Xd[:3].contiguous())
bf.mars_fit(Xd[:2].contiguous(), yd)
bf.rank_similarity(Xd[0, :20].contiguous(), Xd[1, :20].contiguous())
torch.cuda.synchronize()
print("sanitize workload done")
