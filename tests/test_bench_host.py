"""Host-side logic of bench.py (no GPU)."""
import numpy as np
import pytest

import bench
from paper_conf_ipps_stoltzfushsld21_b200 import inputs as I
from paper_conf_ipps_stoltzfushsld21_b200 import rafd


@pytest.mark.parametrize("dims,p", [((20, 16, 40), 2), ((20, 16, 41), 3), ((12, 10, 64), 8), ((9, 7, 16), 4)])
def test_box_plan_matches_library_plan(dims, p):
    nx, ny, nz = dims
    lib_plan = rafd.rafd_slab_plan(I.box_mask(nx, ny, nz).numpy(), 32, 3, p)
    assert bench.slab_plan_box(nx, ny, nz, 32, 3, p) == lib_plan


def test_reference_arm_json_line(monkeypatch):
    class A:
        steps, warmup, config = 2, 1, "C1"
    out = bench.run_reference(A)
    assert out["impl"] == "reference" and out["value"] > 0
    assert out["cpu_baseline"]["kind"] == "oracle"
    assert out["e2e"]["h2d_bytes_per_step"] == 0


class _FakeRoom:
    """Stands in for rafd.Room in the temporal-blocking fallback logic."""
    def __init__(self, fits, n_mask=1 << 30):
        self.fits, self.tb, self.n_mask = fits, 1, n_mask

    def get_info(self):
        return {"n_mask": self.n_mask}

    def set_temporal_blocking(self, n):
        if n == 2 and not self.fits:
            raise rafd.RafdError(rafd.RAFD_E_NOMEM, "cudaMalloc: out of memory")
        self.tb = n


def test_enable_tb_single_rank():
    import torch
    r = _FakeRoom(True)
    assert bench.enable_tb(r, 2, 1, torch.device("cpu")) == 2 and r.tb == 2
    r = _FakeRoom(False)
    assert bench.enable_tb(r, 2, 1, torch.device("cpu")) == 1 and r.tb == 1
    r = _FakeRoom(True)
    assert bench.enable_tb(r, 1, 1, torch.device("cpu")) == 1 and r.tb == 1
    # auto: two steps per sweep from 2^25 voxels on (C3 and up), single steps below (C2)
    assert bench.enable_tb(_FakeRoom(True, 1536 * 1024 * 704), 0, 1, torch.device("cpu")) == 2
    assert bench.enable_tb(_FakeRoom(True, 256 ** 3), 0, 1, torch.device("cpu")) == 1


def _tb_worker(rank, world, port, q):
    import os
    import torch
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        r = _FakeRoom(fits=rank != 1)  # rank 1 runs out of memory
        q.put((rank, bench.enable_tb(r, 2, world, torch.device("cpu")), r.tb))
    finally:
        dist.destroy_process_group()


def test_enable_tb_all_ranks_agree():
    """A NOMEM on one rank turns temporal blocking off on every rank (slabs of
    one room must step with the same steps_per_sweep)."""
    import socket
    import torch.multiprocessing as mp
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_tb_worker, args=(k, 3, port, q)) for k in range(3)]
    for p in procs:
        p.start()
    res = sorted(q.get(timeout=120) for _ in range(3))
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    assert res == [(0, 1, 1), (1, 1, 1), (2, 1, 1)]
