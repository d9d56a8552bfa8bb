"""Thin ctypes binding of librafd.so (include/rafd.h), same names as the C-ABI.

Argument marshalling only: every step of the path runs in the library's CUDA
kernels.  Buffers may be numpy arrays (host) or torch tensors (host or CUDA);
the library copies what it needs before a call returns.  There is no CPU
fallback: loading fails loudly if librafd.so is missing, and rafd_create fails
with RAFD_E_CUDA when no GPU is present.
"""
from __future__ import annotations

import ctypes as C
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "librafd.so")
# A/B experiments: RAFD_LIB points the binding at another build of the same ABI
LIB_PATH = os.environ.get("RAFD_LIB", LIB_PATH)

RAFD_OK = 0
RAFD_E_INVAL = -1
RAFD_E_UNSTABLE = -2
RAFD_E_NONPASSIVE = -3
RAFD_E_OUTSIDE = -4
RAFD_E_MATERIAL = -5
RAFD_E_NOMEM = -6
RAFD_E_CUDA = -7
RAFD_E_NCCL = -8
RAFD_E_STATE = -9
RAFD_SCHEME_TWO_KERNEL = 0
RAFD_SCHEME_LISTING1 = 1
RAFD_SCHEME_NAIVE_FI = 2

# every symbol include/rafd.h declares (checked by tests/test_abi.py)
ABI_SYMBOLS = [
    "rafd_create", "rafd_destroy", "rafd_set_source", "rafd_set_receivers", "rafd_set_state",
    "rafd_step", "rafd_step_group", "rafd_synchronize", "rafd_read_receivers", "rafd_read_field",
    "rafd_read_branch_state", "rafd_get_classification", "rafd_get_info", "rafd_energy",
    "rafd_set_profiling", "rafd_get_kernel_times", "rafd_launch_count", "rafd_slab_plan",
    "rafd_nccl_unique_id", "rafd_last_error", "rafd_strerror", "rafd_version",
    "rafd_ipc_handle", "rafd_ipc_connect", "rafd_set_step", "rafd_set_temporal_blocking",
    "rafd_set_halo_push", "rafd_release_cached_memory",
]
RAFD_IPC_BLOB_BYTES = 352


class rafd_materials(C.Structure):
    _fields_ = [("n_materials", C.c_int32), ("n_branches", C.c_int32),
                ("beta0", C.c_void_p), ("D", C.c_void_p), ("E", C.c_void_p), ("F", C.c_void_p)]


class rafd_room_desc(C.Structure):
    _fields_ = [("nx", C.c_int32), ("ny", C.c_int32), ("nz", C.c_int32),
                ("mask", C.c_void_p), ("matmap", C.c_void_p),
                ("lam", C.c_double), ("precision", C.c_int32),
                ("mat", C.POINTER(rafd_materials)), ("device", C.c_int32),
                ("cuda_stream", C.c_void_p), ("rank", C.c_int32), ("nranks", C.c_int32),
                ("nccl_id", C.c_void_p), ("z_begin", C.c_int32), ("z_end", C.c_int32),
                ("mask_z0", C.c_int32), ("scheme", C.c_int32), ("loss1", C.c_double),
                ("loss2", C.c_double)]


class rafd_info(C.Structure):
    _fields_ = [("n_mask", C.c_int64), ("n_inside", C.c_int64), ("n_boundary", C.c_int64),
                ("k_hist", C.c_int64 * 7), ("isolated", C.c_int64), ("steps", C.c_int64),
                ("bytes_per_step", C.c_int64), ("volume_bytes", C.c_int64),
                ("boundary_bytes", C.c_int64), ("device_bytes", C.c_int64),
                ("precision", C.c_int32), ("n_materials", C.c_int32), ("n_branches", C.c_int32),
                ("z_begin", C.c_int32), ("z_end", C.c_int32), ("pitch", C.c_int32),
                ("fused", C.c_int32), ("scheme", C.c_int32), ("steps_per_sweep", C.c_int32),
                ("reserved_", C.c_int32), ("n_shell", C.c_int64)]


class rafd_kernel_times(C.Structure):
    _fields_ = [("volume_ms", C.c_double), ("boundary_ms", C.c_double), ("other_ms", C.c_double),
                ("volume_launches", C.c_int64), ("boundary_launches", C.c_int64),
                ("other_launches", C.c_int64), ("shell_ms", C.c_double),
                ("shell_launches", C.c_int64)]


_lib = None


def lib():
    """Load librafd.so (raises if it has not been built)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} is missing: build it with "
                          "`python -m paper_conf_ipps_stoltzfushsld21_b200.build` "
                          "(there is no CPU fallback)")
    L = C.CDLL(LIB_PATH)
    P, I32, I64 = C.c_void_p, C.c_int32, C.c_int64
    L.rafd_create.argtypes = [C.POINTER(rafd_room_desc), C.POINTER(P)]
    L.rafd_destroy.argtypes = [P]
    L.rafd_destroy.restype = None
    L.rafd_set_source.argtypes = [P, I32, I32, I32, P, I64]
    L.rafd_set_receivers.argtypes = [P, I32, P]
    L.rafd_set_state.argtypes = [P, P, P, P, P]
    L.rafd_step.argtypes = [P, I64]
    L.rafd_set_temporal_blocking.argtypes = [P, I32]
    L.rafd_set_step.argtypes = [P, I64]
    L.rafd_step_group.argtypes = [C.POINTER(P), I32, I64]
    L.rafd_synchronize.argtypes = [P]
    L.rafd_read_receivers.argtypes = [P, P, I64, C.POINTER(I64)]
    L.rafd_read_field.argtypes = [P, P, P]
    L.rafd_read_branch_state.argtypes = [P, P, P]
    L.rafd_get_classification.argtypes = [P, P, P, P, P]
    L.rafd_get_info.argtypes = [P, C.POINTER(rafd_info)]
    L.rafd_energy.argtypes = [P, C.POINTER(C.c_double)]
    L.rafd_set_profiling.argtypes = [P, C.c_int]
    L.rafd_get_kernel_times.argtypes = [P, C.POINTER(rafd_kernel_times)]
    L.rafd_launch_count.argtypes = [P]
    L.rafd_launch_count.restype = I64
    L.rafd_slab_plan.argtypes = [I32, I32, I32, P, I32, I32, I32, P, P]
    L.rafd_nccl_unique_id.argtypes = [P]
    L.rafd_ipc_handle.argtypes = [P, P]
    L.rafd_ipc_connect.argtypes = [P, P, P]
    L.rafd_set_halo_push.argtypes = [P, I32]
    L.rafd_release_cached_memory.argtypes = [I32]
    L.rafd_last_error.restype = C.c_char_p
    L.rafd_strerror.restype = C.c_char_p
    L.rafd_strerror.argtypes = [C.c_int]
    _lib = L
    return L


class RafdError(RuntimeError):
    def __init__(self, code, msg):
        super().__init__(f"rafd error {code}: {msg}")
        self.code = code


def _check(rc, L=None):
    if rc != RAFD_OK:
        raise RafdError(rc, (L or lib()).rafd_last_error().decode())


def _addr(a):
    """Address of a numpy array or torch tensor (host or device); None for None."""
    if a is None:
        return None
    if hasattr(a, "data_ptr"):
        assert a.is_contiguous(), "tensor must be contiguous"
        return a.data_ptr()
    assert a.flags["C_CONTIGUOUS"], "array must be C-contiguous"
    return a.ctypes.data


def _f64(a, shape=None):
    a = np.ascontiguousarray(a, dtype=np.float64)
    return a if shape is None else a.reshape(shape)


class Room:
    """A room handle (rafd_room*).  Shapes: fields [nz][ny][nx]."""

    def __init__(self, mask, lam, precision, beta0, D=None, E=None, F=None, matmap=None,
                 device=0, stream=None, rank=0, nranks=1, nccl_id=None, z_begin=0, z_end=0,
                 mask_z0=0, dims=None, scheme=0, loss1=1.0, loss2=1.0):
        L = lib()
        # the handle belongs to this library: every method (and __del__) calls
        # it, even if the module is later pointed at another build (RAFD_LIB /
        # the oracle's librafd_oracle.so in tests)
        self._L = L
        # dims = (nx, ny, nz) of the room when `mask` holds only planes [mask_z0, ...)
        nz, ny, nx = (int(s) for s in mask.shape)
        if dims is not None:
            nx, ny, nz = (int(s) for s in dims)
        beta0 = _f64(beta0).reshape(-1)
        M = beta0.size
        if D is None:
            MB = 0
            Dd = Ed = Fd = None
        else:
            Dd = _f64(D).reshape(M, -1)
            MB = Dd.shape[1]
            Ed = _f64(E, (M, MB))
            Fd = _f64(F, (M, MB))
        if hasattr(mask, "data_ptr"):
            assert str(mask.dtype) == "torch.uint8"
        else:
            mask = np.ascontiguousarray(mask, dtype=np.uint8)
        if matmap is not None and not hasattr(matmap, "data_ptr"):
            matmap = np.ascontiguousarray(matmap, dtype=np.uint8)
        self._mat = rafd_materials(M, MB, beta0.ctypes.data,
                                   None if Dd is None else Dd.ctypes.data,
                                   None if Ed is None else Ed.ctypes.data,
                                   None if Fd is None else Fd.ctypes.data)
        idbuf = None
        if nccl_id is not None:
            idbuf = (C.c_uint8 * 128).from_buffer_copy(bytes(nccl_id))
        d = rafd_room_desc(nx, ny, nz, _addr(mask), _addr(matmap), float(lam), int(precision),
                           C.pointer(self._mat), int(device), stream, int(rank), int(nranks),
                           None if idbuf is None else C.addressof(idbuf), int(z_begin), int(z_end),
                           int(mask_z0), int(scheme), float(loss1), float(loss2))
        h = C.c_void_p()
        _check(L.rafd_create(C.byref(d), C.byref(h)), L)
        self.h = h
        self._keep = (mask, matmap, beta0, Dd, Ed, Fd)
        self.shape = (nz, ny, nx)
        self.precision = int(precision)
        self.dtype = np.float32 if precision == 32 else np.float64
        self.M, self.MB = M, MB
        self.nrcv = 0
        info = self.get_info()
        self.z_begin, self.z_end = info["z_begin"], info["z_end"]
        self.nb = info["n_boundary"]

    # --- lifetime
    def destroy(self):
        if getattr(self, "h", None):
            self._L.rafd_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.destroy()
        except Exception:
            pass

    # --- set
    def set_source(self, xyz, sig):
        sig = _f64(sig).reshape(-1)
        _check(self._L.rafd_set_source(self.h, int(xyz[0]), int(xyz[1]), int(xyz[2]),
                                     sig.ctypes.data, sig.size))

    def set_receivers(self, xyzs):
        a = np.ascontiguousarray(np.asarray(xyzs, dtype=np.int32).reshape(-1, 3))
        _check(self._L.rafd_set_receivers(self.h, a.shape[0], a.ctypes.data))
        self.nrcv = a.shape[0]

    def set_state(self, u_prev=None, u_curr=None, v=None, g=None):
        def conv(a):
            if a is None or hasattr(a, "data_ptr"):
                return a
            return np.ascontiguousarray(a, dtype=self.dtype)
        arrs = [conv(a) for a in (u_prev, u_curr, v, g)]
        _check(self._L.rafd_set_state(self.h, *[_addr(a) for a in arrs]))

    def set_step(self, n):
        _check(self._L.rafd_set_step(self.h, int(n)))

    # --- run
    def step(self, n):
        _check(self._L.rafd_step(self.h, int(n)))

    def set_temporal_blocking(self, steps_per_sweep):
        """rafd_set_temporal_blocking: 2 = two leapfrog steps per grid sweep."""
        _check(self._L.rafd_set_temporal_blocking(self.h, int(steps_per_sweep)))

    def synchronize(self):
        _check(self._L.rafd_synchronize(self.h))

    # --- read
    def read_receivers(self, cap=None):
        if self.nrcv == 0:
            return np.zeros((0, 0))
        if cap is None:
            cap = max(1, self.get_info()["steps"])
        out = np.zeros((self.nrcv, cap), dtype=np.float64)
        n = C.c_int64()
        _check(self._L.rafd_read_receivers(self.h, out.ctypes.data, cap, C.byref(n)))
        return out[:, : n.value].copy()

    def read_field(self, out_curr=None, out_prev=None):
        """u^n and u^{n-1} of the owned planes (numpy by default; pass CUDA
        tensors to receive on the device; pass False to skip one)."""
        lnz = self.z_end - self.z_begin
        shp = (lnz, self.shape[1], self.shape[2])
        cur = np.zeros(shp, dtype=self.dtype) if out_curr is None else out_curr
        prv = np.zeros(shp, dtype=self.dtype) if out_prev is None else out_prev
        _check(self._L.rafd_read_field(self.h, None if cur is False else _addr(cur),
                                     None if prv is False else _addr(prv)))
        return (None if cur is False else cur), (None if prv is False else prv)

    def read_branch_state(self):
        v = np.zeros((self.MB, self.nb), dtype=self.dtype)
        g = np.zeros((self.MB, self.nb), dtype=self.dtype)
        _check(self._L.rafd_read_branch_state(self.h, _addr(v), _addr(g)))
        return v, g

    def get_classification(self):
        lnz = self.z_end - self.z_begin
        K = np.zeros((lnz, self.shape[1], self.shape[2]), dtype=np.uint8)
        bidx = np.zeros(self.nb, dtype=np.int64)
        Kb = np.zeros(self.nb, dtype=np.uint8)
        matb = np.zeros(self.nb, dtype=np.uint8)
        _check(self._L.rafd_get_classification(self.h, K.ctypes.data, bidx.ctypes.data,
                                             Kb.ctypes.data, matb.ctypes.data))
        return K, bidx, Kb, matb

    def get_info(self):
        i = rafd_info()
        _check(self._L.rafd_get_info(self.h, C.byref(i)))
        d = {k: getattr(i, k) for k, _ in rafd_info._fields_}
        d["k_hist"] = list(i.k_hist)
        return d

    def energy(self):
        h = C.c_double()
        _check(self._L.rafd_energy(self.h, C.byref(h)))
        return h.value

    def set_profiling(self, on=True):
        _check(self._L.rafd_set_profiling(self.h, 1 if on else 0))

    def get_kernel_times(self):
        t = rafd_kernel_times()
        _check(self._L.rafd_get_kernel_times(self.h, C.byref(t)))
        return {k: getattr(t, k) for k, _ in rafd_kernel_times._fields_}

    def ipc_handle(self):
        """This slab's IPC blob (bytes) for rafd_ipc_connect of its neighbours."""
        buf = (C.c_uint8 * RAFD_IPC_BLOB_BYTES)()
        _check(self._L.rafd_ipc_handle(self.h, buf))
        return bytes(buf)

    def ipc_connect(self, lower, upper):
        lo = None if lower is None else (C.c_uint8 * RAFD_IPC_BLOB_BYTES).from_buffer_copy(lower)
        hi = None if upper is None else (C.c_uint8 * RAFD_IPC_BLOB_BYTES).from_buffer_copy(upper)
        _check(self._L.rafd_ipc_connect(self.h, None if lo is None else C.addressof(lo),
                                      None if hi is None else C.addressof(hi)))

    def set_halo_push(self, on=True):
        """rafd_set_halo_push: the edge-phase kernels store the halo into the
        neighbours' ghost planes (device-initiated) instead of copy pulls."""
        _check(self._L.rafd_set_halo_push(self.h, int(bool(on))))

    def launch_count(self):
        return int(self._L.rafd_launch_count(self.h))


# ------------------------------------------------------------------ C-ABI names
def rafd_create(*a, **k):
    return Room(*a, **k)


def rafd_destroy(room):
    room.destroy()


def rafd_step_group(rooms, nsteps):
    """Step the slabs of one room held by this process (see include/rafd.h)."""
    arr = (C.c_void_p * len(rooms))(*[r.h.value for r in rooms])
    _check(lib().rafd_step_group(arr, len(rooms), int(nsteps)))


def rafd_slab_plan(mask, precision, n_branches, nranks):
    """Cost-weighted z-slab split (host-only, no GPU).  Returns [(z_begin, z_end)]."""
    m = np.ascontiguousarray(mask, dtype=np.uint8)
    nz, ny, nx = m.shape
    zb = np.zeros(nranks, dtype=np.int32)
    ze = np.zeros(nranks, dtype=np.int32)
    _check(lib().rafd_slab_plan(nx, ny, nz, m.ctypes.data, int(precision), int(n_branches),
                                int(nranks), zb.ctypes.data, ze.ctypes.data))
    return list(zip(zb.tolist(), ze.tolist()))


def slab_owner(z, plan):
    """Index of the slab of `plan` [(z_begin, z_end)] that owns plane z."""
    for k, (a, b) in enumerate(plan):
        if a <= z < b:
            return k
    raise ValueError(f"plane {z} outside the plan")


def gather_receivers(per_slab, xyzs, plan):
    """Receiver traces of a slab-decomposed room: row j comes from the slab that
    owns receiver j's plane (the other slabs record +0 there)."""
    out = np.zeros_like(per_slab[0])
    for j, (x, y, z) in enumerate(xyzs):
        out[j] = per_slab[slab_owner(z, plan)][j]
    return out


def rafd_release_cached_memory(device=0):
    """Return the library pool's cached device memory to the driver."""
    _check(lib().rafd_release_cached_memory(int(device)))


def rafd_nccl_unique_id():
    buf = (C.c_uint8 * 128)()
    _check(lib().rafd_nccl_unique_id(buf))
    return bytes(buf)


def rafd_version():
    return int(lib().rafd_version())


def rafd_strerror(code):
    return lib().rafd_strerror(int(code)).decode()
