"""Cross-process z slabs with the IPC transport (rafd_ipc_handle /
rafd_ipc_connect): p processes on one GPU (the same code path drives peer GPUs
over NVLink), blobs exchanged with torch.distributed (gloo), halo planes
pulled by device-to-device copies ordered by GPU-side waits on the
neighbours' signal words, or pushed by the edge-phase kernels themselves into
the neighbours' ghost planes (rafd_set_halo_push, device-initiated).  The
gathered fields, receivers and branch state must equal the undivided room AND
the CPU oracle (SURVEY §8(c) acceptance: multi-GPU vs 1-GPU bitwise, GPU vs
oracle bitwise) bit for bit.

The NCCL send/recv transport (the north_star's) needs one GPU per rank: NCCL
rejects two ranks of one communicator on the same device, so its test runs
only where torch.cuda.device_count() >= world (RAFD_NCCL_SHARED_GPU=1 forces
an attempt on one GPU)."""
import functools
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


@functools.lru_cache(maxsize=None)
def _oracle():
    """Fields, receivers and branch state of the CPU oracle after STEPS steps."""
    from oracle import orc
    mask, mm, beta0, D, E, F, up, uc, src, rcv, sig = _case()
    o = orc.OracleRoom(mask, LAM, 32, beta0, D, E, F, matmap=mm)
    o.set_state(up, uc)
    o.set_source(src, sig)
    o.set_receivers(rcv)
    o.step(STEPS)
    cur, prv = o.read_field()
    v, g = o.read_branch_state()
    return cur, prv, o.read_receivers(), v, g


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, plan, q, push=False, tb=1, transport="ipc"):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_ipps_stoltzfushsld21_b200 import rafd
        dev = rank % torch.cuda.device_count() if transport == "nccl" else 0
        torch.cuda.set_device(dev)
        mask, mm, beta0, D, E, F, up, uc, src, rcv, sig = _case()
        a, b = plan[rank]
        nccl_id = None
        if transport == "nccl":
            ids = [rafd.rafd_nccl_unique_id() if rank == 0 else None]
            dist.broadcast_object_list(ids, src=0)
            nccl_id = ids[0]
        try:
            room = rafd.Room(mask, LAM, 32, beta0, D, E, F, matmap=mm, device=dev, rank=rank, nranks=world,
                             nccl_id=nccl_id, z_begin=a, z_end=b)
            room.set_state(up, uc)
            room.set_source(src, sig)
            room.set_receivers(rcv)
            if tb == 2:
                room.set_temporal_blocking(2)  # before the blob: it carries the second buffer pair
            if transport == "ipc":
                blobs = [None] * world
                dist.all_gather_object(blobs, room.ipc_handle())
                room.ipc_connect(blobs[rank - 1] if rank > 0 else None,
                                 blobs[rank + 1] if rank < world - 1 else None)
                if push:
                    room.set_halo_push(True)
            dist.barrier()
            room.step(STEPS // 2)
            room.step(STEPS - STEPS // 2)
            room.synchronize()
            cur, prv = room.read_field()
            v, g = room.read_branch_state()
            q.put((rank, cur, prv, room.read_receivers(), v, g))
        except Exception as e:  # report instead of hanging the parent
            q.put((rank, None, None, repr(e), None, None))
            raise
        dist.barrier()          # keep buffers mapped until every neighbour is done
        room.destroy()
    finally:
        dist.destroy_process_group()


def _run_slabs(world, push, tb, transport):
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
    vw, gw = whole.read_branch_state()

    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, plan, q, push, tb, transport)) for r in range(world)]
    for p in procs:
        p.start()
    res = dict((r, rest) for r, *rest in (q.get(timeout=180) for _ in range(world)))
    for r in range(world):
        assert res[r][0] is not None, f"rank {r}: {res[r][2]}"
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    cs = np.concatenate([res[r][0] for r in range(world)])
    ps = np.concatenate([res[r][1] for r in range(world)])
    rs = rafd.gather_receivers([res[r][2] for r in range(world)], rcv, plan)
    # each slab holds a contiguous sub-range of the ascending boundary list
    vs = np.concatenate([res[r][3] for r in range(world)], axis=1)
    gs = np.concatenate([res[r][4] for r in range(world)], axis=1)
    # multi-GPU vs 1-GPU: bitwise
    assert np.array_equal(cw, cs)
    assert np.array_equal(pw, ps)
    assert np.array_equal(rw, rs)
    assert np.array_equal(vw, vs) and np.array_equal(gw, gs)
    # and vs the CPU oracle written from the paper: bitwise
    co, po, ro, vo, go = _oracle()
    assert np.array_equal(cs, co)
    assert np.array_equal(ps, po)
    assert np.array_equal(rs, ro)
    assert np.array_equal(vs, vo) and np.array_equal(gs, go)


@pytest.mark.parametrize("world,push,tb", [(w, p, t) for w in (2, 3) for p in (False, True) for t in (1, 2)]
                         + [(5, False, 2), (5, True, 2)])
def test_ipc_slabs_equal_single_room_and_oracle(world, push, tb):
    """tb = 2: temporal blocking in every slab (edge planes single-step, the
    two-step kernel over the interior; two exchanges per double step)."""
    _run_slabs(world, push, tb, "ipc")


@pytest.mark.parametrize("world,tb", [(2, 1), (2, 2), (3, 2)])
def test_nccl_slabs_equal_single_room_and_oracle(world, tb):
    """The NCCL send/recv halo (halo.cu), one GPU per rank."""
    if torch.cuda.device_count() < world and os.environ.get("RAFD_NCCL_SHARED_GPU") != "1":
        pytest.skip(f"NCCL needs one GPU per rank ({torch.cuda.device_count()} < {world})")
    _run_slabs(world, False, tb, "nccl")
