"""ctypes binding of the CPU oracle (liborc.so).

TEST INFRASTRUCTURE ONLY: imported by tests/, __graft_entry__.smoke() and the
cpu_baseline / --impl reference legs of bench.py.  The product package never
imports this module.  See orc.h for what the oracle computes and where the
paper defines it.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "liborc.so")
# the same oracle behind the product's C-ABI names (orc_abi.c)
ABI_LIB_PATH = os.path.join(_HERE, "librafd_oracle.so")
_SOURCES = ["orc.c", "orc_step.inc", "orc.h", "orc_abi.c"]

CFLAGS = ["-std=c11", "-O2", "-ffp-contract=off", "-fopenmp", "-fPIC", "-shared", "-Wall", "-Wextra",
          "-Wno-unused-parameter"]


def build(force: bool = False) -> str:
    """Compile liborc.so (and librafd_oracle.so, the same oracle under the
    product's C-ABI names) with gcc (no FMA contraction, no fast-math)."""
    src_m = max(os.path.getmtime(os.path.join(_HERE, s)) for s in _SOURCES)
    for path, srcs in ((_LIB_PATH, ["orc.c"]), (ABI_LIB_PATH, ["orc.c", "orc_abi.c"])):
        if force or not os.path.exists(path) or os.path.getmtime(path) < src_m:
            tmp = path + f".tmp{os.getpid()}"
            subprocess.check_call(["gcc", *CFLAGS, "-o", tmp, *[os.path.join(_HERE, f) for f in srcs], "-lm"])
            os.replace(tmp, path)
    return _LIB_PATH


class OrcDesc(C.Structure):
    _fields_ = [("nx", C.c_int32), ("ny", C.c_int32), ("nz", C.c_int32),
                ("mask", C.c_void_p), ("matmap", C.c_void_p),
                ("lam", C.c_double), ("precision", C.c_int32),
                ("n_materials", C.c_int32), ("n_branches", C.c_int32),
                ("beta0", C.c_void_p), ("D", C.c_void_p), ("E", C.c_void_p), ("F", C.c_void_p)]


class OrcInfo(C.Structure):
    _fields_ = [("n_mask", C.c_int64), ("n_inside", C.c_int64), ("n_boundary", C.c_int64),
                ("k_hist", C.c_int64 * 7), ("isolated", C.c_int64), ("steps", C.c_int64),
                ("precision", C.c_int32), ("n_materials", C.c_int32), ("n_branches", C.c_int32)]


_lib = None


def lib():
    global _lib
    if _lib is None:
        build()
        L = C.CDLL(_LIB_PATH)
        P = C.c_void_p
        L.orc_create.argtypes = [C.POINTER(OrcDesc), C.POINTER(P)]
        L.orc_create_raw.argtypes = [C.POINTER(OrcDesc), P, P, P, P, P, C.POINTER(P)]
        L.orc_destroy.argtypes = [P]
        L.orc_destroy.restype = None
        L.orc_set_source.argtypes = [P, C.c_int32, C.c_int32, C.c_int32, P, C.c_int64]
        L.orc_set_receivers.argtypes = [P, C.c_int32, P]
        L.orc_set_state.argtypes = [P, P, P, P, P]
        L.orc_step.argtypes = [P, C.c_int64]
        L.orc_set_step.argtypes = [P, C.c_int64]
        L.orc_set_scheme.argtypes = [P, C.c_int32, C.c_double, C.c_double]
        L.orc_read_receivers.argtypes = [P, P, C.c_int64, C.POINTER(C.c_int64)]
        L.orc_read_field.argtypes = [P, P, P]
        L.orc_read_branch_state.argtypes = [P, P, P]
        L.orc_get_classification.argtypes = [P, P, P, P, P]
        L.orc_get_info.argtypes = [P, C.POINTER(OrcInfo)]
        L.orc_energy.argtypes = [P, C.POINTER(C.c_double)]
        L.orc_last_error.restype = C.c_char_p
        L.orc_set_threads.argtypes = [C.c_int32]
        L.orc_get_threads.restype = C.c_int32
        _lib = L
    return _lib


def set_threads(n: int) -> None:
    """OpenMP threads of the oracle's volume / boundary loops (process-wide)."""
    _check(lib().orc_set_threads(int(n)))


def get_threads() -> int:
    return int(lib().orc_get_threads())


class OracleError(RuntimeError):
    def __init__(self, code, msg):
        super().__init__(f"oracle error {code}: {msg}")
        self.code = code


def _check(rc):
    if rc != 0:
        raise OracleError(rc, lib().orc_last_error().decode())


def _ptr(a):
    return None if a is None else a.ctypes.data_as(C.c_void_p)


class OracleRoom:
    """One room in the oracle.  Arrays are numpy; fields are [nz][ny][nx]."""

    def __init__(self, mask, lam, precision, beta0, D=None, E=None, F=None, matmap=None,
                 raw=None):
        mask = np.ascontiguousarray(mask, dtype=np.uint8)
        nz, ny, nx = mask.shape
        beta0 = np.ascontiguousarray(beta0, dtype=np.float64).reshape(-1)
        M = beta0.size
        if D is None:
            MB = 0
        else:
            D = np.ascontiguousarray(D, dtype=np.float64).reshape(M, -1)
            MB = D.shape[1]
            E = np.ascontiguousarray(E, dtype=np.float64).reshape(M, MB)
            F = np.ascontiguousarray(F, dtype=np.float64).reshape(M, MB)
        if raw is not None:
            MB = np.asarray(raw["BI"]).reshape(M, -1).shape[1] if raw.get("BI") is not None else 0
        self._keep = [mask, beta0, D, E, F]
        if matmap is not None:
            matmap = np.ascontiguousarray(matmap, dtype=np.uint8)
            assert matmap.shape == mask.shape
            self._keep.append(matmap)
        d = OrcDesc(nx, ny, nz, mask.ctypes.data, None if matmap is None else matmap.ctypes.data,
                    float(lam), int(precision), M, MB, beta0.ctypes.data,
                    None if D is None else D.ctypes.data, None if E is None else E.ctypes.data,
                    None if F is None else F.ctypes.data)
        h = C.c_void_p()
        if raw is None:
            _check(lib().orc_create(C.byref(d), C.byref(h)))
        else:
            arrs = [np.ascontiguousarray(raw[k], dtype=np.float64).reshape(-1)
                    if raw.get(k) is not None else None for k in ("beta", "BI", "D", "DI", "F")]
            self._keep += arrs
            _check(lib().orc_create_raw(C.byref(d), *[_ptr(a) for a in arrs], C.byref(h)))
        self.h = h
        self.shape = (nz, ny, nx)
        self.precision = int(precision)
        self.dtype = np.float32 if precision == 32 else np.float64
        self.M, self.MB = M, MB
        self.nrcv = 0

    def __del__(self):
        if getattr(self, "h", None):
            lib().orc_destroy(self.h)
            self.h = None

    def info(self):
        i = OrcInfo()
        _check(lib().orc_get_info(self.h, C.byref(i)))
        return {"n_mask": i.n_mask, "n_inside": i.n_inside, "n_boundary": i.n_boundary,
                "k_hist": list(i.k_hist), "isolated": i.isolated, "steps": i.steps}

    @property
    def nb(self):
        return self.info()["n_boundary"]

    def set_source(self, xyz, sig):
        sig = np.ascontiguousarray(sig, dtype=np.float64)
        _check(lib().orc_set_source(self.h, int(xyz[0]), int(xyz[1]), int(xyz[2]),
                                    sig.ctypes.data, sig.size))

    def set_receivers(self, xyzs):
        a = np.ascontiguousarray(np.asarray(xyzs, dtype=np.int32).reshape(-1, 3))
        _check(lib().orc_set_receivers(self.h, a.shape[0], a.ctypes.data))
        self.nrcv = a.shape[0]

    def set_state(self, u_prev=None, u_curr=None, v=None, g=None):
        conv = lambda a: None if a is None else np.ascontiguousarray(a, dtype=self.dtype)
        arrs = [conv(a) for a in (u_prev, u_curr, v, g)]
        _check(lib().orc_set_state(self.h, *[_ptr(a) for a in arrs]))

    def step(self, n):
        _check(lib().orc_step(self.h, int(n)))

    def set_scheme(self, scheme, loss1=1.0, loss2=1.0):
        _check(lib().orc_set_scheme(self.h, int(scheme), float(loss1), float(loss2)))

    def read_receivers(self, cap=None):
        if self.nrcv == 0:
            return np.zeros((0, 0))
        if cap is None:
            cap = self.info()["steps"] + 1
        out = np.zeros((self.nrcv, cap), dtype=np.float64)
        n = C.c_int64()
        _check(lib().orc_read_receivers(self.h, out.ctypes.data, cap, C.byref(n)))
        return out[:, : n.value].copy()

    def read_field(self):
        cur = np.zeros(self.shape, dtype=self.dtype)
        prv = np.zeros(self.shape, dtype=self.dtype)
        _check(lib().orc_read_field(self.h, cur.ctypes.data, prv.ctypes.data))
        return cur, prv

    def read_branch_state(self):
        nb = self.nb
        v = np.zeros((self.MB, nb), dtype=self.dtype)
        g = np.zeros((self.MB, nb), dtype=self.dtype)
        _check(lib().orc_read_branch_state(self.h, _ptr(v), _ptr(g)))
        return v, g

    def classification(self):
        nb = self.nb
        K = np.zeros(self.shape, dtype=np.uint8)
        bidx = np.zeros(nb, dtype=np.int64)
        Kb = np.zeros(nb, dtype=np.uint8)
        matb = np.zeros(nb, dtype=np.uint8)
        _check(lib().orc_get_classification(self.h, K.ctypes.data, bidx.ctypes.data,
                                            Kb.ctypes.data, matb.ctypes.data))
        return K, bidx, Kb, matb

    def energy(self):
        h = C.c_double()
        _check(lib().orc_energy(self.h, C.byref(h)))
        return h.value
