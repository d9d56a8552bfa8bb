"""Cross-process z slabs with the IPC transport (rafd_ipc_handle /
rafd_ipc_connect): p processes on one GPU (the same code path drives peer GPUs
over NVLink), blobs exchanged with torch.distributed (gloo), halo planes
pulled by device-to-device copies ordered by GPU-side waits on the
neighbours' signal words, or pushed by the edge-phase kernels themselves into
the neighbours' ghost planes (rafd_set_halo_push, device-initiated).  The
gathered result must equal the undivided room bit for bit."""
import math
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

pytestmark = pytest.mark.gpu
LAM = 1.0 / math.sqrt(3.0)
DIMS = (40, 34, 30)
STEPS = 61  # the second call is odd: double steps then one single step


def _case():
    from paper_conf_ipps_stoltzfushsld21_b200 import inputs as I
    mask_t = I.dome_mask(*DIMS)
    mm = I.material_map(mask_t, "region", 8).numpy()
    mask = mask_t.numpy()
    beta0, D, E, F = I.fd_tables(8, 3)
    rng = np.random.default_rng(3)
    up = rng.uniform(-1, 1, mask.shape).astype(np.float32)
    uc = rng.uniform(-1, 1, mask.shape).astype(np.float32)
    src = I.source_position(DIMS, mask)
    rcv = I.receiver_positions(DIMS, mask)
    return mask, mm, beta0, D, E, F, up, uc, src, rcv, I.gaussian_pulse(30, 3.0)


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, plan, q, push=False, tb=1):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_ipps_stoltzfushsld21_b200 import rafd
        torch.cuda.set_device(0)
        mask, mm, beta0, D, E, F, up, uc, src, rcv, sig = _case()
        a, b = plan[rank]
        room = rafd.Room(mask, LAM, 32, beta0, D, E, F, matmap=mm, rank=rank, nranks=world, z_begin=a, z_end=b)
        room.set_state(up, uc)
        room.set_source(src, sig)
        room.set_receivers(rcv)
        if tb == 2:
            room.set_temporal_blocking(2)  # before the blob: it carries the second buffer pair
        blobs = [None] * world
        dist.all_gather_object(blobs, room.ipc_handle())
        room.ipc_connect(blobs[rank - 1] if rank > 0 else None, blobs[rank + 1] if rank < world - 1 else None)
        if push:
            room.set_halo_push(True)
        dist.barrier()
        try:
            room.step(STEPS // 2)
            room.step(STEPS - STEPS // 2)
            room.synchronize()
            cur, prv = room.read_field()
            q.put((rank, cur, prv, room.read_receivers()))
        except Exception as e:  # report instead of hanging the parent
            q.put((rank, None, None, repr(e)))
            raise
        dist.barrier()          # keep buffers mapped until every neighbour is done
        room.destroy()
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world,push,tb", [(w, p, t) for w in (2, 3) for p in (False, True) for t in (1, 2)]
                         + [(5, False, 2), (5, True, 2)])
def test_ipc_slabs_equal_single_room(world, push, tb):
    """tb = 2: temporal blocking in every slab (edge planes single-step, the
    two-step kernel over the interior; two exchanges per double step)."""
    from paper_conf_ipps_stoltzfushsld21_b200 import rafd
    mask, mm, beta0, D, E, F, up, uc, src, rcv, sig = _case()
    plan = rafd.rafd_slab_plan(mask, 32, 3, world)
    whole = rafd.Room(mask, LAM, 32, beta0, D, E, F, matmap=mm)
    whole.set_state(up, uc)
    whole.set_source(src, sig)
    whole.set_receivers(rcv)
    whole.step(STEPS)
    cw, pw = whole.read_field()
    rw = whole.read_receivers()

    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, plan, q, push, tb)) for r in range(world)]
    for p in procs:
        p.start()
    res = dict((r, (c, pv, rc)) for r, c, pv, rc in (q.get(timeout=120) for _ in range(world)))
    for r in range(world):
        assert res[r][0] is not None, f"rank {r}: {res[r][2]}"
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    cs = np.concatenate([res[r][0] for r in range(world)])
    ps = np.concatenate([res[r][1] for r in range(world)])
    assert np.array_equal(cw, cs)
    assert np.array_equal(pw, ps)
    rs = rafd.gather_receivers([res[r][2] for r in range(world)], rcv, plan)
    assert np.array_equal(rw, rs)
