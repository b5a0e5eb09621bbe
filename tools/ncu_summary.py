"""Summarise ncu output into profiles/ (run on the GPU box or here).

  python tools/ncu_summary.py launches <launches.csv> <out.txt>
      per-kernel totals of an `ncu --metrics gpu__time_duration.sum` launch list
  python tools/ncu_summary.py full <report.ncu-rep> <out_prefix> [algorithmic bytes per launch]
      key metrics of one `ncu --set full` capture -> <out_prefix>.json / .txt,
      plus the 30 hottest source lines by warp-stall samples
"""
from __future__ import annotations

import csv
import io
import json
import re
import subprocess
import sys
from collections import defaultdict

UNIT = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "KB": 1e3, "MB": 1e6, "GB": 1e9,
        "nsecond": 1e-9, "usecond": 1e-6, "msecond": 1e-3, "second": 1.0, "ns": 1e-9, "us": 1e-6, "ms": 1e-3}

KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "sm__inst_executed.avg.per_cycle_active",
        "smsp__issue_active.avg.pct_of_peak_sustained_active", "lts__t_sector_hit_rate.pct",
        "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum", "launch__registers_per_thread", "launch__grid_size",
        "launch__block_size", "launch__shared_mem_per_block_dynamic", "launch__occupancy_limit_registers",
        "launch__occupancy_limit_shared_mem", "launch__occupancy_limit_warps",
        "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum",
        "l1tex__data_pipe_lsu_wavefronts_mem_shared.avg.pct_of_peak_sustained_elapsed",
        "lts__t_bytes.sum"]


def _num(v: str, unit: str) -> float:
    v = v.replace(",", "")
    try:
        x = float(v)
    except ValueError:
        return float("nan")
    return x * UNIT.get(unit, 1.0)


def launches(path: str, out: str) -> None:
    rows = list(csv.reader(open(path)))
    hdr = None
    tot = defaultdict(lambda: [0, 0.0])
    for r in rows:
        if "Kernel Name" in r and "Metric Value" in r:
            hdr = r
            continue
        if hdr is None or len(r) != len(hdr):
            continue
        d = dict(zip(hdr, r))
        if d.get("Metric Name") != "gpu__time_duration.sum":
            continue
        name = re.sub(r"\(.*", "", d["Kernel Name"]).split("::")[-1][:60]
        t = _num(d["Metric Value"], d.get("Metric Unit", "ns"))
        tot[name][0] += 1
        tot[name][1] += t
    allt = sum(v[1] for v in tot.values()) or 1.0
    lines = [f"# per-kernel totals of {path} (serialised, cold-cache launches under ncu; shares, not absolutes)",
             f"{'kernel':44s} {'launches':>9s} {'total ms':>10s} {'avg us':>10s} {'share':>7s}"]
    for k, (c, t) in sorted(tot.items(), key=lambda kv: -kv[1][1]):
        lines.append(f"{k:44s} {c:9d} {t * 1e3:10.3f} {t / c * 1e6:10.2f} {100 * t / allt:6.1f}%")
    lines.append(f"{'TOTAL':44s} {sum(v[0] for v in tot.values()):9d} {allt * 1e3:10.3f}")
    open(out, "w").write("\n".join(lines) + "\n")
    print("\n".join(lines[:20]))


def full(rep: str, prefix: str, alg_bytes: float | None = None) -> None:
    raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    hdr, units, vals = rows[0], rows[1], rows[2]
    name = re.sub(r"\(.*", "", vals[hdr.index("Kernel Name")]).split("::")[-1] if "Kernel Name" in hdr else rep
    m = {}
    for k in KEYS:
        if k in hdr:
            i = hdr.index(k)
            m[k] = _num(vals[i], units[i])
    dur = m.get("gpu__time_duration.sum", float("nan"))
    traffic = m.get("dram__bytes_read.sum", 0.0) + m.get("dram__bytes_write.sum", 0.0)
    res = {"kernel": name, "report": rep.split("/")[-1], "duration_s": dur, "dram_bytes": traffic,
           "dram_GBps": traffic / dur / 1e9 if dur == dur and dur > 0 else None, "metrics": m}
    if alg_bytes:
        res["algorithmic_bytes"] = alg_bytes
        res["traffic_over_algorithmic"] = traffic / alg_bytes
    # hottest source lines
    src = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass,cuda"],
                         capture_output=True, text=True).stdout
    fname, hot = None, []
    for r in csv.reader(io.StringIO(src)):
        if r and r[0] == "File Path":
            fname = r[1].split("/")[-1]
        elif r and r[0].isdigit() and len(r) > 8 and r[2] == "-":
            try:
                hot.append((fname, int(r[0]), r[1].strip()[:100], int(float(r[4] or 0)), int(float(r[7] or 0))))
            except ValueError:
                pass
    ts = sum(h[3] for h in hot) or 1
    ti = sum(h[4] for h in hot) or 1
    res["hot_lines"] = [{"file": h[0], "line": h[1], "stall_pct": round(100 * h[3] / ts, 2),
                         "inst_pct": round(100 * h[4] / ti, 2), "src": h[2]}
                        for h in sorted(hot, key=lambda h: -h[3])[:30]]
    json.dump(res, open(prefix + ".json", "w"), indent=1)
    lines = [f"# {name}: one launch under ncu --set full --clock-control none ({rep.split('/')[-1]})",
             f"duration {dur * 1e3:.3f} ms; DRAM traffic {traffic / 1e6:.1f} MB"
             + (f" ({res['dram_GBps']:.0f} GB/s)" if res["dram_GBps"] else "")
             + (f"; algorithmic {alg_bytes / 1e6:.1f} MB (traffic/alg = {traffic / alg_bytes:.2f})" if alg_bytes else "")]
    lines += [f"  {k:58s} {v:.4g}" for k, v in m.items()]
    lines.append("hottest source lines (warp-stall samples %, instructions %):")
    lines += [f"  {h['file'][:14]:14s}:{h['line']:<5d} {h['stall_pct']:5.1f}% {h['inst_pct']:5.1f}%  {h['src']}"
              for h in res["hot_lines"]]
    open(prefix + ".txt", "w").write("\n".join(lines) + "\n")
    print("\n".join(lines[:24]))


if __name__ == "__main__":
    if sys.argv[1] == "launches":
        launches(sys.argv[2], sys.argv[3])
    else:
        full(sys.argv[2], sys.argv[3], float(sys.argv[4]) if len(sys.argv) > 4 else None)
