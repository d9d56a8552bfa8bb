"""Benchmark of the FDTD room-acoustics step (volume + FD-MM boundary + source/receivers).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl rafd|reference] [--config C4]

A "step" is one leapfrog time step of the whole hot path (SURVEY §8(a) rows
a2-a6; the once-per-room classification a1 is timed inside `e2e`).  Workload at
N=1: BASELINE.json configs[3], the C4 hall 1536x1024x704 (1.107e9 voxels), box,
FD-MM with 3 branches and 8 materials, fp32; the line also carries
`single_step` (the same room at one step per sweep: Listings 2-4 iterated) and
`strong_t1` (C5, configs[4], on one GPU: T_1 of the strong-scaling curve) and
`fp64` (the C4 room in double precision: the metric is quoted for fp32 and fp64).
N>1 (torchrun, one rank per GPU): C5 2048x1536x2560 (8.05e9 voxels) split into N
z-slabs (rafd_slab_plan; strong scaling, E_p = T_1 / (p T_p)), one-plane halo
exchange per step (NCCL send/recv by default), then a bitwise parity check of
the slab transport against the CPU oracle (`parity`).  `--config C4` at N>1
keeps the earlier weak scaling (704*N planes).  Inputs are synthetic and seeded
(paper_conf_ipps_stoltzfushsld21_b200/inputs.py) and larger than L2.

Prints ONE JSON line on rank 0.  `value` = inside-voxel updates of all ranks /
max-over-ranks device time (CUDA events on the room's stream).
"""
from __future__ import annotations

import argparse
import json
import math
import os
import socket
import subprocess
import sys
import threading
import time

import numpy as np
import torch

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

from paper_conf_ipps_stoltzfushsld21_b200 import inputs as I  # noqa: E402

METRIC = "Gvoxel-updates/s (fp32/fp64) and % of HBM roofline at 1/2/4/8 B200"
UNIT = "Gvox/s"
LAM = 1.0 / math.sqrt(3.0)


def peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


class ClockSampler:
    """nvidia-smi style sampling of SM clocks and throttle reasons via NVML."""

    REASONS = {
        "gpu_idle": 0x1, "applications_clocks_setting": 0x2, "sw_power_cap": 0x4,
        "hw_slowdown": 0x8, "sync_boost": 0x10, "sw_thermal_slowdown": 0x20,
        "hw_thermal_slowdown": 0x40, "hw_power_brake_slowdown": 0x80,
    }

    def __init__(self, device_index):
        self.samples = []
        self.reasons = set()
        self.stop = threading.Event()
        self.ok = False
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(device_index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
            self.ok = True
        except Exception as e:  # pragma: no cover
            self.err = repr(e)

    def _run(self):
        nv = self.nv
        while not self.stop.is_set():
            try:
                self.samples.append(nv.nvmlDeviceGetClockInfo(self.h, nv.NVML_CLOCK_SM))
                r = nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
                for k, bit in self.REASONS.items():
                    if r & bit and k != "gpu_idle":
                        self.reasons.add(k)
            except Exception:
                pass
            time.sleep(0.02)

    def __enter__(self):
        if self.ok:
            self.t = threading.Thread(target=self._run, daemon=True)
            self.t.start()
        return self

    def __exit__(self, *a):
        if self.ok:
            self.stop.set()
            self.t.join()

    def result(self):
        if not self.ok or not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": [], "note": "nvml unavailable"}
        return {"sm_mhz": float(np.median(self.samples)), "sm_max_mhz": float(self.max_mhz),
                "reasons": sorted(self.reasons), "samples": len(self.samples)}


def workload(cfg_name, nranks):
    cfg = dict(I.CONFIGS[cfg_name])
    nx, ny, nz = cfg["dims"]
    if nranks > 1 and cfg_name != "C5" and cfg["shape"] == "box":
        nz = nz * nranks          # weak scaling: one C4-sized slab per GPU
    cfg["room"] = (nx, ny, nz)
    return cfg


def slab_inputs(cfg, z0, z1, device):
    """Box mask + region material map for planes [z0-1, z1] (clipped), generated
    on `device`; returns (mask, matmap, mask_z0)."""
    nx, ny, nz = cfg["room"]
    lo, hi = max(0, z0 - 1), min(nz, z1 + 1)
    if cfg["shape"] != "box":   # non-cuboid configs (C2): whole room, then the slab's planes
        full = I.make_mask(cfg["shape"], nx, ny, nz, device=device)
        mm = I.material_map(full, cfg["rule"], cfg["M"])
        return full[lo:hi].contiguous(), mm[lo:hi].contiguous(), lo
    mask = torch.ones((hi - lo, ny, nx), dtype=torch.uint8, device=device)
    if cfg["rule"] == "region":
        mm = I.region_map_box(nx, ny, nz, lo, hi, M=cfg["M"], device=device)
    else:
        mm = torch.zeros_like(mask)
    return mask, mm, lo


def slab_plan_box(nx, ny, nz, precision, MB, nranks):
    """The cost-weighted split of rafd_slab_plan for a BOX room, from the closed
    form of its per-plane counts (end planes: all boundary; other planes: the
    rim) so the 8e9-voxel mask never has to exist on the host.  Matches
    rafd_slab_plan on boxes (tests/test_bench_host.py)."""
    if nranks == 1:
        return [(0, nz)]
    s = precision // 8
    a, b = nx - 2, ny - 2
    nb_end = nx * ny
    nb_mid = nx * ny - a * b
    c_end = nx * ny + 3 * s * nx * ny + (6 + 3 * s + 4 * s * MB) * nb_end
    c_mid = nx * ny + 3 * s * nx * ny + (6 + 3 * s + 4 * s * MB) * nb_mid
    cost = np.full(nz, float(c_mid))
    cost[0] = cost[-1] = c_end
    pre = np.concatenate([[0.0], np.cumsum(cost)])
    cuts = [0]
    for k in range(1, nranks):
        t = pre[-1] * k / nranks
        e = int(np.searchsorted(pre, t))
        if e > 0 and abs(pre[e - 1] - t) <= abs(pre[e] - t):
            e -= 1
        cuts.append(max(cuts[-1] + 1, min(e, nz - (nranks - k))))
    cuts.append(nz)
    return list(zip(cuts[:-1], cuts[1:]))


def _reduce(t, op):
    """all_reduce a float64 tensor on the process group's device (NCCL: CUDA, gloo: CPU)."""
    if torch.distributed.get_backend() == "nccl":
        t = t.cuda()
    else:
        t = t.cpu()
    torch.distributed.all_reduce(t, op=op)
    return t.cpu()


def bench_device(local_rank):
    """GPU of this rank; RAFD_BENCH_DEVICE pins every rank to one GPU (a
    multi-rank run on a single GPU, IPC transport, for testing)."""
    d = os.environ.get("RAFD_BENCH_DEVICE")
    return int(d) if d is not None else local_rank


def connect_ipc(room, rank, world, push=False):
    """Exchange the slabs' CUDA-IPC blobs and connect neighbours (transports
    'ipc': copy pulls; 'push': the edge-phase kernels store into the
    neighbours' ghost planes)."""
    blobs = [None] * world
    torch.distributed.all_gather_object(blobs, room.ipc_handle())
    room.ipc_connect(blobs[rank - 1] if rank > 0 else None, blobs[rank + 1] if rank < world - 1 else None)
    if push:
        room.set_halo_push(True)
    torch.distributed.barrier()


def make_room(cfg, prec, rank, world, local_rank, transport, stream, tb_want):
    """The room (or this rank's slab of it) of a config, inputs generated on
    the device; temporal blocking enabled as asked (auto: >= 2^25 voxels)."""
    from paper_conf_ipps_stoltzfushsld21_b200 import rafd
    dev = torch.device("cuda", local_rank)
    nx, ny, nz = cfg["room"]
    beta0, D, E, F = I.config_materials(cfg)
    plan = slab_plan_box(nx, ny, nz, prec, cfg["MB"], world)
    z0, z1 = plan[rank]
    nccl_id = _new_nccl_id(world > 1 and transport == "nccl", rank)
    mask, mm, mz0 = slab_inputs(cfg, z0, z1, dev)
    t_c = time.perf_counter()
    room = rafd.Room(mask, LAM, prec, beta0, D, E, F, matmap=mm, device=local_rank,
                     stream=None if stream is None else stream.cuda_stream, rank=rank, nranks=world,
                     nccl_id=nccl_id, z_begin=z0, z_end=z1, mask_z0=mz0, dims=(nx, ny, nz))
    del mask, mm
    torch.cuda.empty_cache()
    # temporal blocking (a slab: edge planes single-step, the interior two-step),
    # before the IPC blob (it carries the second buffer pair)
    tb = enable_tb(room, tb_want, world, dev)
    if world > 1 and transport in ("ipc", "push"):
        connect_ipc(room, rank, world, push=transport == "push")
    t_create = time.perf_counter() - t_c
    mask_np = None if cfg["shape"] == "box" else I.make_mask(cfg["shape"], nx, ny, nz).numpy()
    room.set_source(I.source_position((nx, ny, nz), mask_np), I.impulse())
    room.set_receivers(I.receiver_positions((nx, ny, nz), mask_np))
    return room, tb, t_create, plan


GRAPH_WARM = 32  # untimed steps that instantiate the CUDA graphs of both buffer parities


def time_room(room, steps, warmup, stream, world, clk=None):
    """W untimed warm-up steps (+ GRAPH_WARM more that build the step graphs),
    then K steps between CUDA events on the room's stream (barrier +
    synchronize on both sides): the product path, CUDA graphs of 16 steps.
    Then K more steps launched kernel by kernel with CUDA events around every
    kernel (profiling mode), for the per-kernel times only."""
    import contextlib
    room.step(warmup)
    room.step(GRAPH_WARM)
    room.synchronize()
    room.read_receivers()

    def timed(profile, sampler):
        room.set_profiling(profile)
        n0 = room.launch_count()
        ev0 = torch.cuda.Event(enable_timing=True)
        ev1 = torch.cuda.Event(enable_timing=True)
        if world > 1:
            torch.distributed.barrier()
        torch.cuda.synchronize()
        with (sampler if sampler is not None else contextlib.nullcontext()):
            with torch.cuda.stream(stream):
                ev0.record(stream)
                room.step(steps)
                ev1.record(stream)
            torch.cuda.synchronize()
        if world > 1:
            torch.distributed.barrier()
        kt = room.get_kernel_times() if profile else None
        room.set_profiling(False)
        return ev0.elapsed_time(ev1), room.launch_count() - n0, kt

    ms, launches, _ = timed(False, clk)
    # per-kernel times: the faster of two profiled passes (a single pass is
    # exposed to one-off slowdowns of a few launches)
    ms_prof, _, kt = timed(True, None)
    ms_prof2, _, kt2 = timed(True, None)
    if ms_prof2 < ms_prof:
        ms_prof, kt = ms_prof2, kt2
    kt["profiled_ms"] = ms_prof
    rec = room.read_receivers()
    return ms, launches, kt, rec


def sub_record(room, steps, warmup, stream, prec, tb, peak):
    """One-GPU record of a room at a given steps-per-sweep (the `single_step`
    and `strong_t1` records of the N=1 line)."""
    ms, launches, kt, _ = time_room(room, steps, warmup, stream, 1)
    info = room.get_info()
    s = prec // 8
    vol_bytes = info["volume_bytes"] if tb == 1 else info["n_mask"] + info["n_inside"] * 4 * s
    launch_ms = kt["volume_ms"] / max(1, kt["volume_launches"])
    bnd_launch_ms = kt["boundary_ms"] / max(1, kt["boundary_launches"])
    vol_gbs = vol_bytes / (launch_ms * 1e-3) / 1e9
    return {"value": round(info["n_inside"] * steps / (ms * 1e-3) / 1e9, 3), "unit": UNIT,
            "ms_per_step": round(ms / steps, 4), "steps": steps, "warmup": warmup, "steps_per_sweep": tb,
            "n_inside": info["n_inside"],
            "volume_kernel": "k_volume2 (two steps per sweep)" if tb == 2 else "k_volume_tma",
            "volume_launch_ms": round(launch_ms, 5), "volume_gbs": round(vol_gbs, 1),
            "volume_frac_of_peak": round(vol_gbs / peak, 4),
            "boundary_us_per_launch": round(bnd_launch_ms * 1e3, 2),
            "boundary_gbs": round(info["boundary_bytes"] / (bnd_launch_ms * 1e-3) / 1e9, 1)
            if info["n_boundary"] else None,
            "shell_us_per_step": round(kt["shell_ms"] / steps * 1e3, 2),
            "gpu_launches": int(launches)}


def run_rafd(args, rank, world, local_rank):
    from paper_conf_ipps_stoltzfushsld21_b200 import build
    if rank == 0:
        build.build()
    if world > 1:
        torch.distributed.barrier()
    local_rank = bench_device(local_rank)
    dev = torch.device("cuda", local_rank)
    torch.cuda.set_device(dev)
    cfg = workload(args.config, world)
    nx, ny, nz = cfg["room"]
    prec = cfg["precision"] if args.precision is None else args.precision
    stream = torch.cuda.Stream(device=dev)
    room, tb, t_create, plan = make_room(cfg, prec, rank, world, local_rank, args.transport, stream, args.tb)
    info = room.get_info()
    clk = ClockSampler(local_rank)
    ms, launches, kt, rec = time_room(room, args.steps, args.warmup, stream, world, clk)

    info = room.get_info()
    t = torch.tensor([ms, float(info["n_inside"]), float(info["bytes_per_step"]), float(launches),
                      kt["volume_ms"], kt["boundary_ms"], kt["other_ms"]], dtype=torch.float64,
                     device=dev)
    if world > 1:
        mx = _reduce(t.clone(), torch.distributed.ReduceOp.MAX)
        sm = _reduce(t.clone(), torch.distributed.ReduceOp.SUM)
    else:
        mx = sm = t
    ms_max = float(mx[0])
    n_in_total = float(sm[1])
    bytes_total = float(sm[2])
    value = n_in_total * args.steps / (ms_max * 1e-3) / 1e9
    strong = world > 1 and args.config == "C5"

    out = None
    peak, peak_src = peaks()
    if rank == 0:
        fused = bool(info["fused"])
        # per step: one volume launch per step on one GPU; a slab splits it into
        # edge-plane and interior launches, so sum them per step
        vol_ms = kt["volume_ms"] / args.steps
        bnd_ms = kt["boundary_ms"] / args.steps if kt["boundary_launches"] else 0.0
        # the fused kernel moves the whole step's algorithmic bytes (volume + boundary)
        vol_bytes = info["bytes_per_step"] if fused else info["volume_bytes"]
        n_mask = info["n_mask"]
        if tb == 2:
            # k_volume2 per launch (two steps): reads u^{n-1}, u^n, K, writes u^{n+1}, u^{n+2}
            vol_bytes = n_mask * 1 + info["n_inside"] * 4 * (prec // 8)
        launch_ms = kt["volume_ms"] / max(1, kt["volume_launches"])
        if tb == 2 and world > 1:
            # a slab's double step runs k_volume2 over the interior planes and the
            # single-step kernel twice over the two edge planes: time them together
            # per double step against the two-step algorithmic bytes of the slab
            launch_ms = kt["volume_ms"] / (args.steps / 2)
        vol_gbs = vol_bytes / (launch_ms * 1e-3) / 1e9
        bnd_gbs = info["boundary_bytes"] / (bnd_ms * 1e-3) / 1e9 if (info["n_boundary"] and bnd_ms > 0) else None
        step_gbs = bytes_total * args.steps / (ms_max * 1e-3) / 1e9 / world
        traffic, traffic_src = None, None
        # ncu DRAM bytes of one launch of the timed kernel on this config: a
        # committed `ncu --set full` capture (profiles/), not measured in this run
        tp = os.path.join(ROOT, "profiles", "volume2_traffic.json" if tb == 2 else "volume_traffic.json")
        if os.path.exists(tp):
            try:
                tj = json.load(open(tp))
                if bool(tj.get("fused", False)) == fused and args.config == "C4" and world == 1 \
                        and tj.get("precision", 32) == prec:
                    traffic = tj.get("dram_bytes_per_launch")
                    traffic_src = ("committed constant: ncu --set full capture " + os.path.relpath(tp, ROOT)
                                   + (f" ({tj['source']})" if tj.get("source") else "") + "; not measured in this run")
            except Exception:
                traffic = None
        out = {
            "metric": METRIC, "value": round(value, 3), "unit": UNIT, "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(ms_max / args.steps, 4),
            "higher_is_better": True, "scaling": "strong" if strong else "weak", "vs_baseline": None,
            "dtype": "f32" if prec == 32 else "f64",
            "data": f"synthetic (seeded {cfg['shape']} room, {cfg['rule']} materials, "
                    + ("seeded FD tables" if cfg['MB'] else "FI admittances from absorption") + ", impulse source)",
            "config": {
                "workload": f"{args.config}: {nx}x{ny}x{nz} {cfg['shape']} room, "
                            + (f"FD-MM MB={cfg['MB']}" if cfg['MB'] else "FI-MM") + f" M={cfg['M']}, "
                            f"fp{prec}" + (f", {world} z-slabs" if world > 1 else ""),
                "room_dims_xyz": [nx, ny, nz], "n_inside": int(n_in_total),
                "halo_transport": args.transport if world > 1 else None,
                "n_boundary_rank0": info["n_boundary"], "parallelism": f"z-slab x{world}",
                "l2": "inputs larger than L2 (working set %.1f GB/GPU vs 126 MB L2)" % (info["device_bytes"] / 1e9),
                "timed": "CUDA events on the room stream around K steps replayed from CUDA graphs (the product "
                         "path) after W + %d untimed steps; per-kernel times from K more steps launched with "
                         "events around every kernel (the faster of two such passes)" % GRAPH_WARM,
                "steps_per_sweep": tb,
                # RAFD_BENCH_DEVICE pins every rank to one GPU (a functional check of the
                # multi-rank path): the ranks then share that GPU's bandwidth
                "ranks_per_gpu": world if os.environ.get("RAFD_BENCH_DEVICE") is not None else 1,
            },
            "roofline": {
                "bound": "hbm",
                "kernel": ("k_volume2 (two leapfrog steps per sweep)" + (" + edge-plane k_volume_tma per double step"
                                                                          if world > 1 else "")) if tb == 2 else
                          ("k_volume_tma (volume + fused FD-MM boundary)" if fused else "k_volume_tma"),
                "achieved": round(vol_gbs, 1), "peak": peak,
                "unit": "GB/s", "frac": round(vol_gbs / peak, 4), "traffic": traffic,
                "traffic_source": traffic_src,
                "algorithmic_bytes_per_launch": vol_bytes,
                "avg_launch_ms": round(launch_ms, 5), "launches_per_step": kt["volume_launches"] / args.steps,
                "peak_source": peak_src,
                **({"traffic_frac_of_peak": round(traffic / (launch_ms * 1e-3) / 1e9 / peak, 4),
                    "note": "k_volume2 moves its ncu DRAM traffic (1.04x the algorithmic bytes: overlapped-tile "
                            "re-reads) at traffic_frac_of_peak; capping the persistent grid shows it bound per SM "
                            "(time = ceil(units / CTAs) x 0.19 ms for 100..148 CTAs), "
                            "profiles/r02_volume2_alternatives_ab.txt"}
                   if tb == 2 and world == 1 and traffic else {}),
            },
            "kernels": {
                "volume_ms_per_step": round(vol_ms, 5), "boundary_ms_per_step": round(bnd_ms, 5),
                "other_ms_per_step": round(kt["other_ms"] / args.steps, 5),
                # the same K steps launched kernel by kernel with events around each
                "profiled_ms_per_step": round(kt["profiled_ms"] / args.steps, 5),
                "shell_ms_per_step": round(kt["shell_ms"] / args.steps, 5),
                "n_shell": info["n_shell"],
                "boundary_gbs": None if bnd_gbs is None else round(bnd_gbs, 1),
                "boundary_share": round(bnd_ms / (ms_max / args.steps), 4),
                "fused_boundary": fused,
                # the one-step-per-sweep method's algorithmic bytes (SURVEY §8(d) B_step)
                # per step over the measured time.  An EQUIVALENT bandwidth, not DRAM
                # throughput: with two steps per sweep fewer bytes actually move, so
                # it can exceed the copy peak
                "step_equivalent_gbs_per_gpu": round(step_gbs, 1),
                "step_equivalent_frac_of_peak": round(step_gbs / peak, 4),
            },
            "gpu_launches": int(launches),
            "clocks": clk.result(),
            "create_s": round(t_create, 3),
            "receivers_checksum": float(np.abs(rec).sum()),
        }
    if world == 1 and not args.no_sub_records:
        # the north_star's two-kernel step (Listings 2-4, one step per sweep),
        # measured in the same run on the same room
        if tb == 2:
            room.set_temporal_blocking(1)
            out["single_step"] = sub_record(room, args.steps, args.warmup, stream, prec, 1, peak)
            out["single_step"]["what"] = ("PAPER.md Listings 2-4 iterated (volume kernel + FD-MM boundary "
                                          "kernel per step, source/receivers fused), same room")
    room.destroy()
    del room
    from paper_conf_ipps_stoltzfushsld21_b200 import rafd
    rafd.rafd_release_cached_memory(local_rank)  # the library caches freed rooms; give the memory back
    torch.cuda.synchronize()
    torch.cuda.empty_cache()
    if world == 1 and args.config == "C4" and not args.no_sub_records:
        # C5 (BASELINE configs[4]) on one GPU: T_1 of the strong-scaling curve
        c5 = workload("C5", 1)
        r5, tb5, _, _ = make_room(c5, prec, 0, 1, local_rank, args.transport, stream, args.tb)
        rec5 = sub_record(r5, args.steps, args.warmup, stream, prec, tb5, peak)
        rec5["workload"] = "C5: 2048x1536x2560 box room, FD-MM MB=3 M=8, fp%d, 1 GPU" % prec
        rec5["efficiency_formula"] = ("E_p = T_1 / (p * T_p), T = ms_per_step of C5: this record (p = 1) and "
                                      "`bench.py --gpus p` (C5 split into p z-slabs)")
        out["strong_t1"] = rec5
        r5.destroy()
        del r5
        rafd.rafd_release_cached_memory(local_rank)
        torch.cuda.synchronize()
        torch.cuda.empty_cache()
        # the metric is "Gvoxel-updates/s (fp32/fp64)": the same C4 room in fp64
        if prec == 32:
            r6, tb6, _, _ = make_room(cfg, 64, 0, 1, local_rank, args.transport, stream, args.tb)
            rec6 = sub_record(r6, args.steps, args.warmup, stream, 64, tb6, peak)
            rec6["workload"] = "C4: 1536x1024x704 box room, FD-MM MB=3 M=8, fp64, 1 GPU"
            out["fp64"] = rec6
            r6.destroy()
            del r6
            rafd.rafd_release_cached_memory(local_rank)
            torch.cuda.synchronize()
            torch.cuda.empty_cache()
    e2e = run_e2e(args, cfg, prec, *I.config_materials(cfg), rank, world, local_rank, plan,
                  world > 1 and args.transport == "nccl")
    if rank == 0:
        out["e2e"] = e2e
    if world > 1:
        par = parity_leg(args, rank, world, local_rank)
        if rank == 0:
            out["parity"] = par
    return out


def parity_leg(args, rank, world, local_rank, steps=49):
    """N > 1 self-check, run after the timing: a small non-cuboid FD-MM room
    (dome 96 x 80 x 16N, MB=3, M=8, fp32, random initial field, source and
    receivers) split into the N ranks' z-slabs over the bench's transport,
    stepped with one and with two steps per sweep; fields, branch state and
    receivers gathered on rank 0 and compared bit for bit with the CPU oracle
    (SURVEY §8(c) acceptance)."""
    from paper_conf_ipps_stoltzfushsld21_b200 import rafd
    dims = (96, 80, 16 * world)
    mask_t = I.dome_mask(*dims)
    mask = mask_t.numpy()
    mm = I.material_map(mask_t, "region", 8).numpy()
    beta0, D, E, F = I.fd_tables(8, 3)
    rng = np.random.default_rng(17)
    up = (rng.uniform(-1, 1, mask.shape) * mask).astype(np.float32)
    uc = (rng.uniform(-1, 1, mask.shape) * mask).astype(np.float32)
    src = I.source_position(dims, mask)
    rcv = I.receiver_positions(dims, mask)
    sig = I.gaussian_pulse(40, 4.0)
    plan = rafd.rafd_slab_plan(mask, 32, 3, world)
    z0, z1 = plan[rank]
    res = {"room": "dome %dx%dx%d FD-MM MB=3 M=8 fp32, %d steps" % (dims + (steps,)), "transport": args.transport,
           "slabs": [list(p) for p in plan]}
    ref = None
    if rank == 0:
        from oracle import orc
        o = orc.OracleRoom(mask, LAM, 32, beta0, D, E, F, matmap=mm)
        o.set_state(up, uc)
        o.set_source(src, sig)
        o.set_receivers(rcv)
        o.step(steps)
        ref = (*o.read_field(), *o.read_branch_state(), o.read_receivers())
    ok_all = True
    for tb in (1, 2):
        nccl_id = _new_nccl_id(args.transport == "nccl", rank)
        room = rafd.Room(mask, LAM, 32, beta0, D, E, F, matmap=mm, device=local_rank, rank=rank, nranks=world,
                         nccl_id=nccl_id, z_begin=z0, z_end=z1)
        room.set_state(up, uc)
        room.set_source(src, sig)
        room.set_receivers(rcv)
        if tb == 2:
            room.set_temporal_blocking(2)
        if args.transport in ("ipc", "push"):
            connect_ipc(room, rank, world, push=args.transport == "push")
        room.step(steps // 2)
        room.step(steps - steps // 2)
        room.synchronize()
        cur, prv = room.read_field()
        v, g = room.read_branch_state()
        rec = room.read_receivers()
        parts = [None] * world
        torch.distributed.all_gather_object(parts, (cur, prv, v, g, rec))
        torch.distributed.barrier()  # IPC: keep the buffers mapped until every neighbour is done
        room.destroy()
        if rank == 0:
            got = (np.concatenate([q[0] for q in parts]), np.concatenate([q[1] for q in parts]),
                   np.concatenate([q[2] for q in parts], axis=1), np.concatenate([q[3] for q in parts], axis=1),
                   rafd.gather_receivers([q[4] for q in parts], rcv, plan))
            eq = [bool(np.array_equal(a, b)) for a, b in zip(got, ref)]
            res[f"bitwise_tb{tb}"] = dict(zip(["u_n", "u_n_minus_1", "v", "g", "receivers"], eq))
            ok_all = ok_all and all(eq)
    if rank == 0:
        res["parity_ok"] = ok_all
        log = os.environ.get("NCCL_DEBUG_FILE", "")
        if log:
            path = log.replace("%h", socket.gethostname()).replace("%p", str(os.getpid()))
            try:
                lines = [ln.strip() for ln in open(path) if "Init COMPLETE" in ln or "nranks" in ln]
                res["nccl_comm_lines"] = lines[-8:]
                res["comm_nranks_ok"] = any(f"nranks {world} " in ln for ln in lines)
            except OSError as e:
                res["nccl_comm_lines"] = [f"no NCCL debug log ({e})"]
    return res


def enable_tb(room, want, world, dev):
    """Two leapfrog steps per sweep when asked for and the second buffer pair
    fits (C5 fp32 on one GPU needs ~143 GB); every rank must run the same
    setting, so a NOMEM anywhere falls back to single steps everywhere."""
    from paper_conf_ipps_stoltzfushsld21_b200 import rafd
    if want == 0:
        info = room.get_info()
        want = 2 if info["n_mask"] >= (1 << 25) else 1
        if world > 1:  # every rank decides alike (slabs of one room share the setting)
            t = torch.tensor([want], dtype=torch.int32, device=dev)
            torch.distributed.all_reduce(t, op=torch.distributed.ReduceOp.MIN)
            want = int(t[0])
    tb = 1
    if want == 2:
        try:
            room.set_temporal_blocking(2)
            tb = 2
        except rafd.RafdError as e:
            if e.code != rafd.RAFD_E_NOMEM:
                raise
            print(f"temporal blocking does not fit ({e}); single steps", file=sys.stderr)
    if world > 1:
        t = torch.tensor([tb], dtype=torch.int32, device=dev)
        torch.distributed.all_reduce(t, op=torch.distributed.ReduceOp.MIN)
        if int(t[0]) != tb:
            room.set_temporal_blocking(1)
            tb = 1
    return tb


E2E_REPS = 3


def _new_nccl_id(multi, rank):
    if not multi:
        return None
    from paper_conf_ipps_stoltzfushsld21_b200 import rafd
    obj = [rafd.rafd_nccl_unique_id() if rank == 0 else None]
    torch.distributed.broadcast_object_list(obj, src=0)
    return obj[0]


def _e2e_once(args, cfg, prec, beta0, D, E, F, rank, world, local_rank, plan, mask_h, mm_h, mz0, nccl_id, ipc, sig,
              mask_np, rcv, steps, rafd):
    """One end-to-end run (create .. destroy); returns (max wall over ranks, inside voxels, D2H bytes, steps per call)."""
    nx, ny, nz = cfg["room"]
    z0, z1 = plan[rank]
    if world > 1:
        torch.distributed.barrier()
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    room = rafd.Room(mask_h.numpy(), LAM, prec, beta0, D, E, F, matmap=mm_h.numpy(), device=local_rank,
                     rank=rank, nranks=world, nccl_id=nccl_id, z_begin=z0, z_end=z1, mask_z0=mz0,
                     dims=(nx, ny, nz))
    tb = enable_tb(room, args.tb, world, torch.device("cuda", local_rank))
    if ipc:
        connect_ipc(room, rank, world, push=args.transport == "push")
    room.set_source(I.source_position((nx, ny, nz), mask_np), sig)
    room.set_receivers(rcv)
    d2h = 0
    done = 0
    while done < steps:
        k = min(tb, steps - done)  # a double step with temporal blocking: read both samples
        room.step(k)
        r = room.read_receivers(cap=k)
        d2h += r.shape[0] * r.shape[1] * (prec // 8)
        done += k
    room.synchronize()
    t1 = time.perf_counter()
    n_in = room.get_info()["n_inside"]
    room.destroy()
    el = torch.tensor([t1 - t0, float(n_in)], dtype=torch.float64, device=torch.device("cuda", local_rank))
    if world > 1:
        mx = _reduce(el.clone(), torch.distributed.ReduceOp.MAX)
        sm = _reduce(el.clone(), torch.distributed.ReduceOp.SUM)
        tmax, n_tot = float(mx[0]), float(sm[1])
    else:
        tmax, n_tot = float(el[0]), float(el[1])
    return tmax, n_tot, d2h, tb


def run_e2e(args, cfg, prec, beta0, D, E, F, rank, world, local_rank, plan, multi):
    """End to end through the public API with HOST buffers: create the room from
    pinned host mask/matmap (H2D + on-device classification), set source and
    receivers, then every step: rafd_step(1) and rafd_read_receivers (D2H of the
    step's receiver samples); destroy.  Wall clock, max over ranks; the median
    of E2E_REPS runs (allocating and freeing the room's ~20 GB varies by up to
    0.6 s from run to run, tools/e2e_phases.py)."""
    from paper_conf_ipps_stoltzfushsld21_b200 import rafd
    nx, ny, nz = cfg["room"]
    z0, z1 = plan[rank]
    local_rank = bench_device(local_rank)
    mask_d, mm_d, mz0 = slab_inputs(cfg, z0, z1, torch.device("cuda", local_rank))
    mask_h = torch.empty(mask_d.shape, dtype=torch.uint8, pin_memory=True)
    mm_h = torch.empty(mm_d.shape, dtype=torch.uint8, pin_memory=True)
    mask_h.copy_(mask_d)
    mm_h.copy_(mm_d)
    del mask_d, mm_d
    torch.cuda.empty_cache()
    nccl_id = None
    if multi:
        obj = [rafd.rafd_nccl_unique_id() if rank == 0 else None]
        torch.distributed.broadcast_object_list(obj, src=0)
        nccl_id = obj[0]
    ipc = world > 1 and args.transport in ("ipc", "push")
    sig = I.impulse()
    mask_np = None if cfg["shape"] == "box" else I.make_mask(cfg["shape"], nx, ny, nz).numpy()
    rcv = I.receiver_positions((nx, ny, nz), mask_np)
    steps = args.steps
    walls = []
    rafd.rafd_release_cached_memory(local_rank)  # the first run allocates from the driver (cold)
    for _rep in range(E2E_REPS):
        tmax, n_tot, d2h, tb = _e2e_once(args, cfg, prec, beta0, D, E, F, rank, world, local_rank, plan, mask_h, mm_h,
                                         mz0, nccl_id if _rep == 0 else _new_nccl_id(multi, rank), ipc, sig, mask_np,
                                         rcv, steps, rafd)
        walls.append(tmax)
    tmax = sorted(walls)[len(walls) // 2]  # median run: cudaMalloc/cudaFree of the room's ~20 GB vary run to run
    h2d = mask_h.numel() + mm_h.numel() + sig.size * 8
    return {"value": round(n_tot * steps / tmax / 1e9, 3), "unit": UNIT,
            "h2d_bytes_per_step": int(h2d // steps), "d2h_bytes_per_step": int(d2h // steps),
            "wall_s": round(tmax, 3), "wall_s_runs": [round(w, 3) for w in walls],
            "cold_wall_s": round(walls[0], 3),
            "h2d_bytes_note": "the input tensors handed to rafd_create (mask, matmap) and the source signal; "
                              "the library moves the mask over PCIe bit-packed (host threads pack it: 1/8 of "
                              "its bytes) and reads the matmap only at boundary nodes",
            "includes": "rafd_create from pinned host mask+matmap (H2D, device classification), "
                        "set_source/set_receivers, per step rafd_step(1)+rafd_read_receivers (D2H), destroy; "
                        "median of %d runs (the first allocates from the driver, later ones reuse the library's "
                        "memory cache)" % E2E_REPS
                        + ("; temporal blocking: rafd_step(2) + a read of both samples per call" if tb == 2 else "")}


def oracle_sample(cfg, nplanes):
    """Bounded sample of the workload for the CPU oracle: the same x-y section,
    `nplanes` planes (a box of nx x ny x nplanes), same materials."""
    from oracle import orc
    nx, ny, nz = cfg["room"]
    if cfg["shape"] == "box":
        mask = I.box_mask(nx, ny, nplanes)
    else:  # a slice of planes from the middle of the non-cuboid room
        z0 = max(0, nz // 2 - nplanes // 2)
        mask = I.make_mask(cfg["shape"], nx, ny, nz)[z0:z0 + nplanes].contiguous()
    mm = I.material_map(mask, cfg["rule"], cfg["M"]).numpy()
    beta0, D, E, F = I.config_materials(cfg)
    prec = cfg["precision"]
    r = orc.OracleRoom(mask.numpy(), LAM, prec, beta0, D, E, F, matmap=mm)
    m = mask.numpy()
    r.set_source(I.source_position((nx, ny, nplanes), m), I.impulse())
    r.set_receivers(I.receiver_positions((nx, ny, nplanes), m))
    return r, (nx, ny, nplanes)


def cpu_model():
    try:
        for ln in open("/proc/cpuinfo"):
            if ln.startswith("model name"):
                return ln.split(":", 1)[1].strip()
    except OSError:
        pass
    import platform
    return platform.processor() or "unknown"


def host_cores():
    try:
        return len(os.sched_getaffinity(0))
    except AttributeError:
        return os.cpu_count() or 1


def _time_oracle(cfg, threads, seconds, nplanes):
    from oracle import orc
    orc.set_threads(threads)
    r, dims = oracle_sample(cfg, nplanes)
    n_in = r.info()["n_inside"]
    r.step(1)
    t0 = time.perf_counter()
    n = 0
    while time.perf_counter() - t0 < seconds:
        r.step(1)
        n += 1
    dt = time.perf_counter() - t0
    return n_in * n / dt / 1e9, n, dt, dims


def cpu_baseline(cfg, seconds=8.0):
    """The oracle as it stands (OpenMP over z planes and boundary nodes, results
    independent of the thread count) on a bounded sample of the workload: at
    all host cores (`value`, `cores`) and single-threaded (`single_thread`)."""
    cores = host_cores()
    # OpenMP splits the volume loop over z planes: give every thread two planes
    nplanes = max(16, min(256, 2 * cores))
    v_n, n_n, dt_n, dims_n = _time_oracle(cfg, cores, seconds, nplanes)
    v_1, n_1, dt_1, dims_1 = _time_oracle(cfg, 1, seconds, 16)
    from oracle import orc
    orc.set_threads(cores)
    crop = lambda d: f"{d[0]}x{d[1]}x{d[2]} box crop of the workload (same x-y section and materials)"
    return {"value": round(v_n, 5), "unit": UNIT, "cores": cores, "kind": "oracle",
            "sample": f"{crop(dims_n)}, {n_n} steps in {dt_n:.1f} s, C oracle (-O2 -ffp-contract=off "
                      f"-fopenmp, {cores} threads)",
            "cpu_model": cpu_model(),
            "single_thread": {"value": round(v_1, 5), "unit": UNIT, "cores": 1,
                              "sample": f"{crop(dims_1)}, {n_1} steps in {dt_1:.1f} s"}}


def run_reference(args):
    """--impl reference: the CPU oracle as it stands (the only reference this
    tier has) on all host cores, each step a bounded sample of the workload."""
    from oracle import orc
    cfg = workload(args.config, 1)
    cores = host_cores()
    orc.set_threads(cores)
    nplanes = max(16, min(256, 2 * cores))
    r, dims = oracle_sample(cfg, nplanes)
    n_in = r.info()["n_inside"]
    r.step(args.warmup)
    t0 = time.perf_counter()
    r.step(args.steps)
    dt = time.perf_counter() - t0
    v = n_in * args.steps / dt / 1e9
    sample = f"{dims[0]}x{dims[1]}x{dims[2]} box crop of {args.config} (same x-y section and materials)"
    return {"impl": "reference", "metric": METRIC, "value": round(v, 5), "unit": UNIT, "n_gpus": 0,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(dt / args.steps * 1e3, 3),
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None,
            "dtype": "f32" if cfg["precision"] == 32 else "f64", "data": "synthetic",
            "config": {"workload": f"{args.config} sample: {sample}"},
            "cpu_baseline": {"value": round(v, 5), "unit": UNIT, "cores": cores, "kind": "oracle",
                             "sample": sample + f", C oracle with OpenMP ({cores} threads)",
                             "cpu_model": cpu_model()},
            "e2e": {"value": round(v, 5), "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=200)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="rafd", choices=["rafd", "reference"])
    ap.add_argument("--config", default=None,
                    help="default: C4 at N=1 (BASELINE configs[3]); C5 split into N z-slabs at N>1 "
                         "(configs[4], strong scaling)")
    ap.add_argument("--precision", type=int, default=None)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-sub-records", action="store_true",
                    help="N=1: skip the single_step (C4, one step per sweep), strong_t1 (C5 on one GPU) and fp64 (C4) records")
    ap.add_argument("--tb", type=int, default=0, choices=[0, 1, 2],
                    help="steps per HBM sweep (2: temporal blocking); 0 = auto: 2 for rooms of >= 2^25 "
                         "voxels per GPU, 1 below (measured: C2 256^3 is faster with single steps, C3 and "
                         "up with two, profiles/r01_other_configs.txt)")
    ap.add_argument("--transport", default="nccl", choices=["nccl", "ipc", "push"],
                    help="halo exchange for --gpus > 1: NCCL send/recv, or CUDA-IPC peer copies "
                         "ordered by GPU-side stream waits (rafd_ipc_connect)")
    args = ap.parse_args()
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    if args.config is None:
        args.config = "C5" if world > 1 and args.impl != "reference" else "C4"
    if world > 1 and "NCCL_DEBUG" not in os.environ:
        # communicator init lines (nranks, devices) for the parity record, in a file:
        # stdout carries only the JSON line
        os.environ.update(NCCL_DEBUG="INFO", NCCL_DEBUG_SUBSYS="INIT",
                          NCCL_DEBUG_FILE="/tmp/rafd_nccl.%h.%p.log")
    if args.impl == "reference":
        if rank == 0:  # the oracle is a CPU program: rank 0 alone runs it
            print(json.dumps(run_reference(args)), flush=True)
        return
    if world > 1:
        dev = bench_device(local_rank)
        torch.cuda.set_device(dev)
        if args.transport == "nccl":
            torch.distributed.init_process_group("nccl", device_id=torch.device("cuda", dev))
        else:  # IPC halo: the process group only carries the blobs and the timing reductions
            torch.distributed.init_process_group("gloo")
    out = run_rafd(args, rank, world, local_rank)
    if rank == 0:
        if world == 1 and not args.no_cpu_baseline:
            out["cpu_baseline"] = cpu_baseline(workload(args.config, 1))
        else:
            out["cpu_baseline"] = None
        print(json.dumps(out), flush=True)
    if world > 1:
        torch.distributed.barrier()
        torch.distributed.destroy_process_group()


if __name__ == "__main__":
    main()
