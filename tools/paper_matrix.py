"""The paper's experiment matrix on a B200.

Table II rooms (602x402x302, 336^3, 302x202x152; box exact, dome with our own
generator -- the paper's dome geometry is not given, R12) x FI-MM /
FD-MM (MB=3) x single / double precision.  For each cell: the volume kernel,
the boundary kernel alone (the quantity of the paper's Tables V and VI) and
the whole step, timed with CUDA events around every launch (rafd profiling
mode) over `--steps` steps after `--warmup`.  The paper's best time for the
same cell (any of its four GPUs, OpenCL or LIFT; tools/paper_tables.json,
PAPER.md:1685-1823) is printed beside it: context on other hardware, not a
target.  Writes profiles/<tag>_paper_matrix.{json,md}.

    python tools/paper_matrix.py [--steps 50] [--warmup 5] [--tag r01]
"""
import argparse
import json
import math
import os
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_ipps_stoltzfushsld21_b200 import inputs as I, rafd  # noqa: E402

LAM = 1.0 / math.sqrt(3.0)


def paper_best(tables, key, size, shape, prec):
    rows = [r for r in tables[key] if r["size"] == size and r["shape"] == shape]
    if not rows:
        return None
    f = "sp_ms" if prec == 32 else "dp_ms"
    b = min(rows, key=lambda r: r[f])
    return {"ms": b[f], "gpu": f"{b['platform']} {b['version']}", "line": b["paper_line"]}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--steps", type=int, default=50)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--tag", default="r01")
    a = ap.parse_args()
    tables = json.load(open(os.path.join(ROOT, "tools", "paper_tables.json")))
    dev = torch.device("cuda", 0)
    out = []
    for size, dims in tables["sizes"].items():
        nx, ny, nz = dims
        for shape in ("box", "dome"):
            mask = I.make_mask(shape, nx, ny, nz, device=dev)
            mm = I.material_map(mask, "region", 8)
            for kind, MB in (("FI-MM", 0), ("FD-MM", 3)):
                if MB:
                    beta0, D, E, F = I.fd_tables(8, 3)
                else:
                    beta0, D, E, F = I.fi_beta_from_alpha([0.05, 0.2, 0.5, 0.9, 0.3, 0.1, 0.7, 0.4]), None, None, None
                for prec in (32, 64):
                    r = rafd.Room(mask, LAM, prec, beta0, D, E, F, matmap=mm)
                    info = r.get_info()
                    r.set_source(I.source_position((nx, ny, nz), mask.cpu().numpy()), I.impulse())
                    r.step(a.warmup)
                    r.synchronize()
                    r.set_profiling(True)
                    r.step(a.steps)
                    kt = r.get_kernel_times()
                    r.set_profiling(False)
                    vol = kt["volume_ms"] / kt["volume_launches"]
                    bnd = kt["boundary_ms"] / max(1, kt["boundary_launches"])
                    oth = kt["other_ms"] / max(1, kt["other_launches"])
                    step = vol + bnd + oth
                    # the same room with temporal blocking (two steps per sweep)
                    r.set_temporal_blocking(2)
                    r.step(2 * (a.warmup // 2 + 1))
                    r.synchronize()
                    r.set_profiling(True)
                    n2 = 2 * (a.steps // 2)
                    r.step(n2)
                    k2 = r.get_kernel_times()
                    r.set_profiling(False)
                    step2 = (k2["volume_ms"] + k2["boundary_ms"] + k2["other_ms"] + k2["shell_ms"]) / n2
                    nb, nin = info["n_boundary"], info["n_inside"]
                    key = "table_v_fimm_boundary_only" if MB == 0 else "table_vi_fdmm_mb3_boundary_only"
                    pb = paper_best(tables, key, int(size), shape, prec)
                    pv = paper_best(tables, "table_iv_fi_naive_one_kernel", int(size), "box", prec) \
                        if (shape == "box" and MB == 0) else None
                    row = {"room": f"{nx}x{ny}x{nz}", "shape": shape, "boundary": kind, "precision": prec,
                           "n_inside": nin, "n_boundary": nb,
                           "volume_ms": round(vol, 4), "boundary_ms": round(bnd, 4), "step_ms": round(step, 4),
                           "step_gvox_s": round(nin / (step * 1e-3) / 1e9, 2),
                           "volume_gvox_s": round(nin / (vol * 1e-3) / 1e9, 2),
                           "boundary_gpts_s": round(nb / (bnd * 1e-3) / 1e9, 2),
                           "step_algorithmic_gbs": round(info["bytes_per_step"] / (step * 1e-3) / 1e9, 1),
                           "tb2_step_ms": round(step2, 4), "tb2_step_gvox_s": round(nin / (step2 * 1e-3) / 1e9, 2),
                           "paper_boundary_best": pb, "paper_fi_one_kernel_best": pv}
                    if pb:
                        row["boundary_speedup_vs_paper_best"] = round(pb["ms"] / bnd, 1)
                    if pv:
                        row["step_speedup_vs_paper_fi_one_kernel"] = round(pv["ms"] / step, 1)
                    out.append(row)
                    print(json.dumps(row), flush=True)
                    r.destroy()
                    del r
                    torch.cuda.empty_cache()
            # Table IV's kernel itself: the naive one-kernel FI of Listing 6 (scheme 2), box only
            if shape == "box":
                for prec in (32, 64):
                    c = 0.1
                    r = rafd.Room(mask, LAM, prec, [0.0], scheme=2, loss1=1 / (1 + c), loss2=1 - c)
                    nin = r.get_info()["n_inside"]
                    r.set_source(I.source_position((nx, ny, nz)), I.impulse())
                    r.step(a.warmup)
                    r.synchronize()
                    r.set_profiling(True)
                    r.step(a.steps)
                    kt = r.get_kernel_times()
                    r.set_profiling(False)
                    vol = kt["volume_ms"] / kt["volume_launches"]
                    pv = paper_best(tables, "table_iv_fi_naive_one_kernel", int(size), "box", prec)
                    row = {"room": f"{nx}x{ny}x{nz}", "shape": shape, "boundary": "naive FI (Listing 6, 1 kernel)",
                           "precision": prec, "n_inside": nin, "n_boundary": r.get_info()["n_boundary"],
                           "volume_ms": round(vol, 4), "boundary_ms": 0.0, "step_ms": round(vol, 4),
                           "step_gvox_s": round(nin / (vol * 1e-3) / 1e9, 2), "volume_gvox_s": round(nin / (vol * 1e-3) / 1e9, 2),
                           "boundary_gpts_s": None, "step_algorithmic_gbs": round(nin * (1 + 3 * prec // 8) / (vol * 1e-3) / 1e9, 1),
                           "paper_boundary_best": None, "paper_fi_one_kernel_best": pv,
                           "kernel_speedup_vs_paper_table_iv": round(pv["ms"] / vol, 1)}
                    out.append(row)
                    print(json.dumps(row), flush=True)
                    r.destroy()
                    del r
                    torch.cuda.empty_cache()
            del mask, mm
    os.makedirs(os.path.join(ROOT, "profiles"), exist_ok=True)
    json.dump(out, open(os.path.join(ROOT, "profiles", f"{a.tag}_paper_matrix.json"), "w"), indent=1)
    lines = ["| room | shape | boundary | prec | Nb | volume ms | boundary ms (Gpts/s) | step ms (Gvox/s) | "
             "step ms, 2 steps/sweep (Gvox/s) | paper best boundary ms (GPU, PAPER.md line) | "
             "paper best FI one-kernel ms |",
             "|---|---|---|---|---|---|---|---|---|---|---|"]
    for r in out:
        pb = r["paper_boundary_best"]
        pv = r["paper_fi_one_kernel_best"]
        lines.append(f"| {r['room']} | {r['shape']} | {r['boundary']} | fp{r['precision']} | {r['n_boundary']} | "
                     f"{r['volume_ms']} | " + (f"{r['boundary_ms']} ({r['boundary_gpts_s']})" if r['boundary_gpts_s'] else "—") +
                     f" | {r['step_ms']} ({r['step_gvox_s']}) | "
                     + (f"{r['tb2_step_ms']} ({r['tb2_step_gvox_s']})" if r.get('tb2_step_ms') else "—") + " | "
                     + (f"{pb['ms']} ({pb['gpu']}, {pb['line']})" if pb else "—") + " | "
                     + (f"{pv['ms']} ({pv['gpu']}, {pv['line']})" if pv else "—") + " |")
    open(os.path.join(ROOT, "profiles", f"{a.tag}_paper_matrix.md"), "w").write(
        "# The paper's experiment matrix on one B200 (context: the paper's numbers are other GPUs)\n\n"
        "Dome rows use this build's dome (DESIGN.md R12), not the paper's (its boundary counts differ).\n"
        "Times: CUDA events around each launch, mean over the timed steps.  '2 steps/sweep': the same\n"
        "room with temporal blocking (k_volume2 + boundary + shell + source per step, DESIGN.md §6).\n"
        "The boundary kernel also injects the source and records the receivers in its last block\n"
        "(whole-room steps, DESIGN.md §6): its column includes that tail (~2 us).\n\n" + "\n".join(lines) + "\n")


if __name__ == "__main__":
    main()
