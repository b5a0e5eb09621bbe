"""bench.py contract checks that need no GPU: both arms print BASELINE.json's metric (so the driver's
reference ratio is defined), and `--gpus N` without WORLD_SIZE re-launches itself under
torch.distributed.run with N ranks (rank 0 alone prints; the reference arm runs the CPU oracle)."""
from __future__ import annotations

import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_metric_is_baselines():
    sys.path.insert(0, ROOT)
    import bench
    base = json.load(open(os.path.join(ROOT, "BASELINE.json")))
    assert bench.METRIC == base["metric"]


def test_gpus_flag_spawns_ranks_reference_arm():
    env = {k: v for k, v in os.environ.items() if k not in ("WORLD_SIZE", "RANK", "LOCAL_RANK")}
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference", "--config", "C1",
                        "--gpus", "2", "--steps", "1", "--warmup", "0"], cwd=ROOT, env=env, capture_output=True,
                       text=True, timeout=600)
    assert r.returncode == 0, r.stderr[-2000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, r.stdout[-2000:]          # rank 0 alone prints
    d = json.loads(lines[0])
    assert d["impl"] == "reference" and d["n_gpus"] == 2
    assert d["metric"] == json.load(open(os.path.join(ROOT, "BASELINE.json")))["metric"]
    assert d["e2e"]["h2d_bytes_per_step"] == 0 and d["cpu_baseline"]["kind"] == "oracle"


def test_ncu_summary_picks_the_newest_profile_round():
    """The roofline's `traffic` comes from the newest committed ncu summary: profile directories are ordered by
    round, then suffix length, then suffix (r02z < r02aa), not by name."""
    import importlib.util
    import re
    spec = importlib.util.spec_from_file_location("bench_mod", os.path.join(ROOT, "bench.py"))
    mod = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(mod)
    d, src = mod._ncu_summary("k_subtree", "C4")
    assert d is not None and src is not None
    have = [x for x in os.listdir(os.path.join(ROOT, "profiles"))
            if os.path.exists(os.path.join(ROOT, "profiles", x, "full_k_subtree.json"))]

    def key(x):
        m = re.match(r"r(\d+)([a-z]*)$", x)
        return (int(m.group(1)), len(m.group(2)), m.group(2))
    assert src.split(os.sep)[1] == max(have, key=key)
