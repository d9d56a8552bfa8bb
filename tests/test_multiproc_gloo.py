"""World-size-2 CPU tests (gloo) of the multi-process host logic that bench.py
and a user of the multi-GPU path run before any kernel: the slab plan every
rank computes independently, the NCCL-id broadcast, each rank's slab inputs
(owned planes + ghost planes, generated locally with mask_z0), and the
owner-based receiver gather.  The device side of the slab decomposition is
covered bitwise on one GPU by tests/test_gpu_slabs.py."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import bench
from paper_conf_ipps_stoltzfushsld21_b200 import inputs as I
from paper_conf_ipps_stoltzfushsld21_b200 import rafd


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), RANK=str(rank), WORLD_SIZE=str(world))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        res = {}
        cfg = bench.workload("C3", world)              # 512x384x(256*world) box, weak scaling
        nx, ny, nz = cfg["room"]
        res["room"] = cfg["room"]
        plan = bench.slab_plan_box(nx, ny, nz, 32, cfg["MB"], world)
        plans = [None] * world
        dist.all_gather_object(plans, plan)
        res["plans_agree"] = all(p == plans[0] for p in plans)
        res["plan"] = plan
        # rank 0's id reaches every rank unchanged (a fake id: libnccl is not needed here)
        obj = [bytes(range(128)) if rank == 0 else None]
        dist.broadcast_object_list(obj, src=0)
        res["id_ok"] = obj[0] == bytes(range(128))
        # slab inputs: planes [z0-1, z1] of the whole room
        z0, z1 = plan[rank]
        mask, mm, lo = bench.slab_inputs(cfg, z0, z1, torch.device("cpu"))
        full_mm = I.region_map_box(nx, ny, nz, max(0, z0 - 1), min(nz, z1 + 1), M=cfg["M"])
        res["inputs_ok"] = bool(torch.equal(mm, full_mm)) and lo == max(0, z0 - 1) and \
            mask.shape[0] == min(nz, z1 + 1) - lo
        # owned planes of all ranks tile the room exactly
        owned = [None] * world
        dist.all_gather_object(owned, (z0, z1))
        res["tiles"] = sorted(owned) == [(a, b) for a, b in plan] and owned[0][0] == 0 and owned[-1][1] == nz
        # receiver gather: each rank records its own receivers, +0 elsewhere
        rcv = I.receiver_positions((nx, ny, nz))
        mine = np.zeros((len(rcv), 5))
        for j, (x, y, z) in enumerate(rcv):
            if z0 <= z < z1:
                mine[j] = 1000 * j + np.arange(5)
        per = [None] * world
        dist.all_gather_object(per, mine)
        got = rafd.gather_receivers(per, rcv, plan)
        res["rcv_ok"] = bool(np.array_equal(got, 1000 * np.arange(len(rcv))[:, None] + np.arange(5)))
        # max-over-ranks timing reduction used by bench.py
        t = torch.tensor([1.0 + rank, 10.0 * (rank + 1)], dtype=torch.float64)
        mx = t.clone()
        dist.all_reduce(mx, op=dist.ReduceOp.MAX)
        sm = t.clone()
        dist.all_reduce(sm, op=dist.ReduceOp.SUM)
        res["reduce_ok"] = float(mx[0]) == float(world) and float(sm[1]) == 10.0 * world * (world + 1) / 2
        q.put((rank, res))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2])
def test_multiprocess_host_logic_gloo(world):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    out = dict(q.get(timeout=240) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    for r in range(world):
        res = out[r]
        assert res["plans_agree"] and res["id_ok"] and res["inputs_ok"], res
        assert res["tiles"] and res["rcv_ok"] and res["reduce_ok"], res
    nz = out[0]["room"][2]
    sizes = [b - a for a, b in out[0]["plan"]]
    assert sum(sizes) == nz and abs(sizes[0] - sizes[1]) <= 2
