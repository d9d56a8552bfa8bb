"""The method's PLAIN DEFINITION, written out independently of the oracle, used
only to pin the oracle (tests/test_oracle_pins.py).

For every inside voxel i, with du = u+ - u-  (R5):

    u+ - 2u + u-  =  l^2 sum_{j in N(i)} (u_j - u_i)
                     - l (6 - |N(i)|) [ beta0 du/2 + sum_b (v'_b + v_b)/2 ]
    branch b:  2D (v' - v) + E (v' + v) + 2F g' = du,   g' = g + (v' + v)/2

N(i) is enumerated from the mask with an explicit adjacency list (no K array,
no boundary list).  Each boundary voxel's (1+MB) unknowns (u+, v'_b) are
obtained from a dense linear solve; interior voxels (|N(i)| = 6) are explicit.
Everything in float64.  This is a different algorithm from Listings 2-4 (a
linear solve instead of the closed-form elimination, neighbour sums from an
adjacency list), so agreement to rounding pins the listings' algebra.
"""
from __future__ import annotations

import numpy as np


class PlainFVTD:
    def __init__(self, mask, lam, beta0, D=None, E=None, F=None, matmap=None):
        mask = np.asarray(mask).astype(bool)
        nz, ny, nx = mask.shape
        self.shape = mask.shape
        coords = np.argwhere(mask)                    # (z, y, x) of mask voxels
        index = -np.ones(mask.shape, dtype=np.int64)
        index[tuple(coords.T)] = np.arange(len(coords))
        # explicit adjacency list over mask voxels
        nbrs = [[] for _ in range(len(coords))]
        for k, (z, y, x) in enumerate(coords):
            for dz, dy, dx in ((1, 0, 0), (-1, 0, 0), (0, 1, 0), (0, -1, 0), (0, 0, 1), (0, 0, -1)):
                zz, yy, xx = z + dz, y + dy, x + dx
                if 0 <= zz < nz and 0 <= yy < ny and 0 <= xx < nx and mask[zz, yy, xx]:
                    nbrs[k].append(index[zz, yy, xx])
        deg = np.array([len(n) for n in nbrs])
        keep = deg > 0                                 # isolated voxels are outside
        self.coords = coords[keep]
        remap = -np.ones(len(coords), dtype=np.int64)
        remap[keep] = np.arange(keep.sum())
        self.nbrs = [remap[np.array(n, dtype=np.int64)] for n, k in zip(nbrs, keep) if k]
        self.deg = deg[keep]
        self.n = len(self.coords)
        self.lam = float(lam)
        self.beta0 = np.asarray(beta0, dtype=np.float64).reshape(-1)
        M = self.beta0.size
        if D is None:
            self.MB = 0
            self.D = self.E = self.F = np.zeros((M, 0))
        else:
            self.D = np.asarray(D, dtype=np.float64).reshape(M, -1)
            self.MB = self.D.shape[1]
            self.E = np.asarray(E, dtype=np.float64).reshape(M, self.MB)
            self.F = np.asarray(F, dtype=np.float64).reshape(M, self.MB)
        mm = np.zeros(mask.shape, dtype=np.int64) if matmap is None else np.asarray(matmap, dtype=np.int64)
        self.mat = mm[tuple(self.coords.T)]
        self.bnd = np.flatnonzero(self.deg < 6)        # boundary voxels, ascending canonical order
        self.u = np.zeros(self.n)
        self.um = np.zeros(self.n)
        self.v = np.zeros((self.MB, len(self.bnd)))
        self.g = np.zeros((self.MB, len(self.bnd)))

    def canonical(self):
        nz, ny, nx = self.shape
        z, y, x = self.coords.T
        return (z * ny + y) * nx + x

    def set_fields(self, u_prev, u_curr):
        self.um = np.asarray(u_prev, dtype=np.float64)[tuple(self.coords.T)].copy()
        self.u = np.asarray(u_curr, dtype=np.float64)[tuple(self.coords.T)].copy()

    def field(self, vec):
        out = np.zeros(self.shape)
        out[tuple(self.coords.T)] = vec
        return out

    def step(self, src=None, amp=0.0):
        lam, u, um = self.lam, self.u, self.um
        lap = np.array([u[nb].sum() - len(nb) * u[i] for i, nb in enumerate(self.nbrs)])
        up = 2 * u - um + lam * lam * lap                      # interior (|N|=6) update
        vnew = np.zeros_like(self.v)
        gnew = np.zeros_like(self.g)
        MB = self.MB
        for k, i in enumerate(self.bnd):
            a = 6 - self.deg[i]
            m = self.mat[i]
            b0 = self.beta0[m]
            D, E, F = self.D[m], self.E[m], self.F[m]
            A = np.zeros((MB + 1, MB + 1))
            rhs = np.zeros(MB + 1)
            A[0, 0] = 1 + lam * a * b0 / 2
            A[0, 1:] = lam * a / 2
            rhs[0] = up[i] + lam * a * b0 * um[i] / 2 - lam * a * self.v[:, k].sum() / 2
            for b in range(MB):
                A[1 + b, 0] = -1.0
                A[1 + b, 1 + b] = 2 * D[b] + E[b] + F[b]
                rhs[1 + b] = -um[i] + (2 * D[b] - E[b] - F[b]) * self.v[b, k] - 2 * F[b] * self.g[b, k]
                if A[1 + b, 1 + b] == 0.0:                    # unused (padded) branch: v' = 0
                    A[1 + b, :] = 0.0
                    A[1 + b, 1 + b] = 1.0
                    rhs[1 + b] = 0.0
            sol = np.linalg.solve(A, rhs)
            up[i] = sol[0]
            vnew[:, k] = sol[1:]
            gnew[:, k] = self.g[:, k] + (sol[1:] + self.v[:, k]) / 2
        if src is not None:
            up[src] += amp
        self.um, self.u = u, up
        self.v, self.g = vnew, gnew
