"""C-ABI checks that need no GPU: the library builds, loads and exports every
symbol include/rafd.h declares; host-only helpers work; create fails loudly
(no CPU fallback) when no CUDA device is present."""
import ctypes
import os
import re

import numpy as np
import pytest
import torch

from paper_conf_ipps_stoltzfushsld21_b200 import build, rafd
from paper_conf_ipps_stoltzfushsld21_b200 import inputs as I

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def L():
    build.build()
    return rafd.lib()


def declared_symbols():
    src = open(os.path.join(ROOT, "include", "rafd.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(rafd_[a-z_0-9]+)\s*\(", src)))


def test_header_symbols_exported(L):
    decl = declared_symbols()
    assert len(decl) >= 20
    for name in decl:
        assert hasattr(L, name), name
    assert sorted(rafd.ABI_SYMBOLS) == decl


def test_exports_are_c_symbols():
    out = os.popen(f"nm -D --defined-only {rafd.LIB_PATH}").read()
    for name in declared_symbols():
        assert re.search(rf"\bT {name}$", out, re.M), name


def test_version_and_strerror(L):
    assert rafd.rafd_version() == 1
    assert "outside" in rafd.rafd_strerror(rafd.RAFD_E_OUTSIDE)


def test_binary_is_sm100a():
    out = os.popen(f"/usr/local/cuda/bin/cuobjdump --list-elf {rafd.LIB_PATH}").read()
    assert "sm_100a" in out


def test_library_never_links_the_oracle():
    out = os.popen(f"ldd {rafd.LIB_PATH}").read() + os.popen(f"nm -D {rafd.LIB_PATH}").read()
    assert "orc" not in out.replace("__orc", "")
    csrc = os.path.join(ROOT, "paper_conf_ipps_stoltzfushsld21_b200", "csrc")
    for f in os.listdir(csrc):
        txt = open(os.path.join(csrc, f)).read()
        assert "oracle" not in txt and "orc.h" not in txt, f


@pytest.mark.skipif(torch.cuda.is_available(), reason="checks the no-GPU failure path")
def test_create_without_gpu_fails_loudly(L):
    with pytest.raises(rafd.RafdError) as e:
        rafd.Room(np.ones((4, 4, 4), np.uint8), 0.5, 32, [0.0])
    assert e.value.code == rafd.RAFD_E_CUDA


def test_validation_before_device(L):
    m = np.ones((4, 4, 4), np.uint8)
    with pytest.raises(rafd.RafdError) as e:
        rafd.Room(m, 0.6, 32, [0.0])
    assert e.value.code == rafd.RAFD_E_UNSTABLE
    with pytest.raises(rafd.RafdError) as e:
        rafd.Room(m, 0.5, 16, [0.0])
    assert e.value.code == rafd.RAFD_E_INVAL
    with pytest.raises(rafd.RafdError) as e:
        rafd.Room(m, 0.5, 32, [0.0], D=[[1.0]], E=[[-1.0]], F=[[0.0]])
    assert e.value.code == rafd.RAFD_E_NONPASSIVE


def plane_costs(mask, s, MB):
    p = np.pad(mask.astype(np.int32), 1)
    K = (p[:-2, 1:-1, 1:-1] + p[2:, 1:-1, 1:-1] + p[1:-1, :-2, 1:-1] + p[1:-1, 2:, 1:-1] +
         p[1:-1, 1:-1, :-2] + p[1:-1, 1:-1, 2:]) * mask
    nin = (K > 0).sum(axis=(1, 2))
    nb = ((K > 0) & (K < 6)).sum(axis=(1, 2))
    return mask.shape[1] * mask.shape[2] + 3 * s * nin + (6 + 3 * s + 4 * s * MB) * nb


def test_slab_plan_balances_cost(L):
    mask = I.box_mask(40, 30, 64).numpy()
    for p in (1, 2, 3, 4, 8):
        plan = rafd.rafd_slab_plan(mask, 32, 3, p)
        assert plan[0][0] == 0 and plan[-1][1] == 64
        for (a, b), (c, d) in zip(plan, plan[1:]):
            assert b == c and a < b
        # each slab's cost is within one plane's cost of the ideal share
        c = plane_costs(mask, 4, 3)
        ideal = c.sum() / p
        for a, b in plan:
            assert abs(c[a:b].sum() - ideal) <= c.max() + 1e-9
    # a dome: the top is sparse, so upper slabs get more planes
    dome = I.dome_mask(48, 48, 64).numpy()
    plan = rafd.rafd_slab_plan(dome, 32, 3, 4)
    sizes = [b - a for a, b in plan]
    assert sizes[-1] > sizes[0]
    with pytest.raises(rafd.RafdError):
        rafd.rafd_slab_plan(mask, 32, 3, 65)


def test_nccl_unique_id_via_dlopen(L):
    """The library dlopens libnccl for the multi-GPU halo and hands out the
    128-byte unique id rank 0 broadcasts (no GPU needed for the id)."""
    try:
        a = rafd.rafd_nccl_unique_id()
        b = rafd.rafd_nccl_unique_id()
    except rafd.RafdError as e:
        pytest.skip(f"libnccl not usable here: {e}")
    assert len(a) == 128 and len(b) == 128 and a != b


def test_slab_and_ipc_entry_points_reject_misuse(L):
    # no GPU needed: argument checks happen before any device work
    assert rafd.lib().rafd_ipc_handle(None, None) == rafd.RAFD_E_INVAL
    assert rafd.lib().rafd_ipc_connect(None, None, None) == rafd.RAFD_E_INVAL
    assert rafd.lib().rafd_step_group(None, 0, 1) == rafd.RAFD_E_INVAL
    assert rafd.lib().rafd_step(None, 1) == rafd.RAFD_E_INVAL
