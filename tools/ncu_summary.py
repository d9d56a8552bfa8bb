"""Summarise ncu captures for profiles/ (run here, no GPU needed).

    python tools/ncu_summary.py launches <launches.csv>      # per-kernel share of the step
    python tools/ncu_summary.py full <report.ncu-rep> [name]  # key metrics of one capture
"""
import csv
import io
import json
import re
import subprocess
import sys
from collections import defaultdict

KEYS = [
    "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
    "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "lts__t_sector_hit_rate.pct",
    "sm__throughput.avg.pct_of_peak_sustained_elapsed", "sm__warps_active.avg.pct_of_peak_sustained_active",
    "launch__registers_per_thread", "launch__grid_size", "launch__block_size",
    "launch__occupancy_limit_shared_mem", "launch__shared_mem_per_block_dynamic",
    "lts__t_bytes.sum", "l1tex__t_bytes.sum",
    "smsp__pcsamp_warps_issue_stalled_long_scoreboard", "smsp__pcsamp_warps_issue_stalled_barrier",
    "smsp__pcsamp_warps_issue_stalled_wait", "smsp__pcsamp_warps_issue_stalled_short_scoreboard",
    "smsp__pcsamp_warps_issue_stalled_selected", "smsp__pcsamp_warps_issue_stalled_not_selected",
    "smsp__pcsamp_warps_issue_stalled_branch_resolving", "smsp__pcsamp_warps_issue_stalled_lg_throttle",
]


def launches(path):
    rows = list(csv.reader(open(path)))
    hdr = None
    per = defaultdict(list)
    order = []
    for r in rows:
        if "Kernel Name" in r:
            hdr = r
            continue
        if hdr and len(r) == len(hdr):
            d = dict(zip(hdr, r))
            name = re.sub(r"\(.*", "", d["Kernel Name"]).replace("void ", "").replace("rafd::", "")
            ns = float(d["Metric Value"]) * (1e3 if d["Metric Unit"] == "usecond" else 1e6 if d["Metric Unit"] == "msecond" else 1)
            per[name].append(ns)
            order.append(name)
    step = [k for k in per if k.startswith(("k_volume", "k_boundary", "k_src", "k_shell<", "k_shell_bnd<"))]
    tot = sum(sum(per[k]) for k in step)
    out = {"kernels": {}, "note": "ncu --metrics gpu__time_duration.sum --clock-control none: cold-cache, serialised; compare shares"}
    for k in step:
        out["kernels"][k] = {"launches": len(per[k]), "avg_us": round(sum(per[k]) / len(per[k]) / 1e3, 3),
                             "share_of_step_kernels": round(sum(per[k]) / tot, 4)}
    other = {k: len(v) for k, v in per.items() if k not in step}
    out["other_kernels(launch counts)"] = other
    return out


def full(path, match=None):
    """Key metrics of the first capture whose kernel name contains `match`."""
    raw = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    r = list(csv.reader(io.StringIO(raw)))
    h, units = r[0], r[1]
    rows = r[2:]
    if match:
        rows = [v for v in rows if match in v[h.index("Kernel Name")]]
    v = rows[0]
    out = {"kernel": v[h.index("Kernel Name")] if "Kernel Name" in h else None, "source": path.split("/")[-1]}
    for k in KEYS:
        if k in h:
            i = h.index(k)
            out[k] = f"{v[i]} {units[i]}".strip()
    return out


if __name__ == "__main__":
    mode, path = sys.argv[1], sys.argv[2]
    match = sys.argv[3] if len(sys.argv) > 3 else None
    print(json.dumps(launches(path) if mode == "launches" else full(path, match), indent=1))
