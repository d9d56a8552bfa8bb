/*
 * rafd.h -- C-ABI of the B200-native room-acoustics FDTD library (librafd.so).
 *
 * One room = a voxelised 3-D grid stepped by the two-kernel leapfrog scheme of
 * Stoltzfus et al., IPDPS'21 (PAPER.md = /root/reference/PAPER.md):
 *   volume kernel    PAPER.md:349-357 (Listing 2, kernel 1)
 *   FI-MM boundary   PAPER.md:371-381 (Listing 3)
 *   FD-MM boundary   PAPER.md:415-442 (Listing 4)
 *   iteration        PAPER.md:850-889 (Listing 5: "the two kernels are executed iteratively")
 * Readings of ambiguous passages are numbered R1..R16 in DESIGN.md §3.
 *
 * Conventions for every function:
 *   - returns RAFD_OK (0) or a negative RAFD_E_* code; rafd_last_error() then
 *     holds a thread-local message;
 *   - "host or device" pointers: the library inspects the pointer
 *     (cudaPointerGetAttributes) and copies from/to either; the CALLER KEEPS
 *     OWNERSHIP of every buffer it passes and may free it after the call returns;
 *   - field arrays are [nz][ny][nx] with x fastest; the canonical voxel index is
 *     (z*ny + y)*nx + x over the room (mask) dims (reading R2);
 *   - T is float for precision 32 and double for precision 64;
 *   - a handle is not thread-safe; distinct handles are independent;
 *   - all work is enqueued on the room's CUDA stream; functions that return
 *     data to the host synchronise that stream.
 * There is no CPU fallback: without a CUDA device every create fails with
 * RAFD_E_CUDA.
 */
#ifndef RAFD_H
#define RAFD_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define RAFD_VERSION 1

#define RAFD_OK 0
#define RAFD_E_INVAL -1      /* null pointer, bad size, bad precision, bad cap            */
#define RAFD_E_UNSTABLE -2   /* lambda <= 0 or lambda^2 > 1/3 (+4 ulp)  (reading R1)      */
#define RAFD_E_NONPASSIVE -3 /* beta0/D/E/F negative or non-finite (reading R5)           */
#define RAFD_E_OUTSIDE -4    /* source / receiver not at an inside voxel (K > 0)          */
#define RAFD_E_MATERIAL -5   /* matmap >= n_materials at a boundary node (reading R4)     */
#define RAFD_E_NOMEM -6      /* device or host allocation failed                           */
#define RAFD_E_CUDA -7       /* CUDA runtime error (message in rafd_last_error)           */
#define RAFD_E_NCCL -8       /* NCCL error or NCCL library not loadable                    */
#define RAFD_E_STATE -9      /* call not valid in the current state                        */

#define RAFD_SCHEME_TWO_KERNEL 0
#define RAFD_SCHEME_LISTING1 1
#define RAFD_SCHEME_NAIVE_FI 2

#define RAFD_MAX_BRANCHES 8
#define RAFD_MAX_MATERIALS 256

typedef struct rafd_room rafd_room;

/* Per-material boundary description (Listings 3-4).
 * n_branches = 0  : FI-MM, admittance beta[m] = beta0[m] (Listing 3).
 * n_branches = MB : FD-MM with MB ODE branches; the library derives, in double
 *                   and in this order (reading R5):
 *                     BI[m][b] = 1/((2D + E) + F)   (0 if D = E = F = 0: padded branch)
 *                     DI[m][b] = (2D - E) - F
 *                     beta[m]  = ((beta0[m] + BI[m][0]) + BI[m][1]) + ...
 *                   and rounds each once to T.
 * Arrays are read during rafd_create only. */
typedef struct rafd_materials {
    int32_t n_materials;     /* M, 1..256                                   */
    int32_t n_branches;      /* MB, 0..8                                    */
    const double *beta0;     /* [M], finite, >= 0                           */
    const double *D, *E, *F; /* [M*MB] row-major [m][b], finite, >= 0       */
} rafd_materials;

typedef struct rafd_room_desc {
    int32_t nx, ny, nz;      /* room (mask) dims, each >= 1; the library adds a 1-voxel halo */
    const uint8_t *mask;     /* host or device [nz][ny][nx]; nonzero = inside               */
    const uint8_t *matmap;   /* host or device [nz][ny][nx] material ids, read only at       */
                             /* boundary nodes; NULL => material 0 everywhere               */
    double lambda;           /* Courant number (PAPER.md "l"), 0 < lambda^2 <= 1/3           */
    int32_t precision;       /* 32 or 64                                                     */
    const rafd_materials *mat;
    int32_t device;          /* CUDA device ordinal                                          */
    void *cuda_stream;       /* cudaStream_t to enqueue on, or NULL for a library stream     */
    /* z-slab decomposition.  nranks <= 1: the whole room on one GPU.
     * nranks > 1: this handle owns planes [z_begin, z_end) of the room (from
     * rafd_slab_plan) and exchanges one halo plane with ranks +-1 every step
     * over NCCL; every rank passes the same mask/matmap/materials. */
    int32_t rank, nranks;
    const uint8_t *nccl_id;  /* 128-byte ncclUniqueId from rafd_nccl_unique_id (rank 0); NULL for */
                             /* slabs held by one process and stepped with rafd_step_group      */
    int32_t z_begin, z_end;
    /* mask / matmap hold planes [mask_z0, ...) of the room (0: the whole room).
     * A slab handle reads planes [z_begin-1, z_end] (clipped to the room), so a
     * rank may pass only those. */
    int32_t mask_z0;
    /* Update scheme (readings R17 in DESIGN.md):
     *  RAFD_SCHEME_TWO_KERNEL (0, default): Listings 2-4, any n_materials / n_branches;
     *  RAFD_SCHEME_LISTING1  (1): the single kernel of Listing 1
     *     with nbrs looked up and one admittance: n_materials = 1,
     *     n_branches = 0, beta = beta0[0]; equal to scheme 0 up to rounding;
     *  RAFD_SCHEME_NAIVE_FI  (2): Listing 6, the naive single
     *     kernel: boundary points scale by the constants loss1, loss2
     *     (next = loss1*((2-l2 K)u + l2 s - loss2*prev)); n_branches = 0, materials unused. */
    int32_t scheme;
    double loss1, loss2;
} rafd_room_desc;

typedef struct rafd_info {
    int64_t n_mask;          /* nx*ny*nz (of this handle's slab)                        */
    int64_t n_inside;        /* voxels with K > 0                                      */
    int64_t n_boundary;      /* Nb: voxels with 0 < K < 6            */
    int64_t k_hist[7];       /* voxel count per K value                                */
    int64_t isolated;        /* mask voxels with no inside neighbour (K = 0, reading R3) */
    int64_t steps;           /* steps taken                                            */
    int64_t bytes_per_step;  /* algorithmic HBM bytes per step           */
    int64_t volume_bytes;    /* ... of which the volume kernel                         */
    int64_t boundary_bytes;  /* ... of which the boundary kernel                       */
    int64_t device_bytes;    /* device memory held by the handle                       */
    int32_t precision, n_materials, n_branches;
    int32_t z_begin, z_end;  /* planes owned                                           */
    int32_t pitch;           /* padded x pitch in elements                              */
    int32_t fused;           /* 1: the boundary update runs inside the volume kernel     */
    int32_t scheme;          /* RAFD_SCHEME_*                                          */
    int32_t steps_per_sweep; /* 1, or 2 with temporal blocking (rafd_set_temporal_blocking) */
    int32_t reserved_;
    int64_t n_shell;         /* voxels recomputed after the boundary update (temporal blocking) */
} rafd_info;

/* Per-kernel device times accumulated while profiling is on (CUDA events on
 * the room's stream around every launch; rafd_step then launches kernels one
 * by one instead of replaying a CUDA graph). */
typedef struct rafd_kernel_times {
    double volume_ms, boundary_ms, other_ms;
    int64_t volume_launches, boundary_launches, other_launches;
    double shell_ms;         /* the shell recompute of temporal blocking */
    int64_t shell_launches;
} rafd_kernel_times;

/* Create a room: validates lambda / tables / dims, copies mask and matmap to
 * the device, classifies voxels on the device (K, ascending boundary list,
 * K_b, mat_b: PAPER.md:306-323, 390-393, 411-412), allocates and zeroes the
 * two field buffers, the boundary-node ring u_b and the branch state.  A host
 * mask is read by host threads (one per core, up to 32) that pack it to one
 * bit per voxel in a process-wide pinned buffer before the copy (environment
 * RAFD_MASK_BITS=0: copy the bytes); a host matmap is read in place at the
 * boundary nodes (pinned) or streamed (pageable).  The inputs are only read,
 * and not used after the call returns.  Errors: INVAL, UNSTABLE,
 * NONPASSIVE, MATERIAL, NOMEM, CUDA, NCCL.  *out is NULL on error. */
int rafd_create(const rafd_room_desc *d, rafd_room **out);

/* Free everything; NULL-safe. */
void rafd_destroy(rafd_room *r);

/* One soft source at global voxel (x,y,z): sig[n] is added to u^{n+1}[src]
 * after the boundary update of step n, counted from the room's creation
 * (reading R10); zero after len samples.  sig: host, double, copied and
 * rounded once to T.  OUTSIDE if K = 0 there.  len = 0 removes the source. */
int rafd_set_source(rafd_room *r, int32_t x, int32_t y, int32_t z, const double *sig, int64_t len);

/* n receivers at global voxels xyz[3*j..3*j+2] (host int32); every step
 * records u^{n+1} at each receiver after the source injection.  Discards
 * unread samples.  OUTSIDE if any K = 0. */
int rafd_set_receivers(rafd_room *r, int32_t n, const int32_t *xyz);

/* Initial state.  u_prev = u^{n-1}, u_curr = u^n: host or device, T-typed
 * [nz][ny][nx] of the whole room (a slab handle reads its planes); values at
 * outside voxels are ignored and stored as +0.  v, g: host or device, T-typed
 * [MB][Nb] branch state (ci = b*Nb + i).  NULL => unchanged.
 * Device inputs (here and in rafd_create) may have been produced on any of the
 * caller's streams: the call first waits for the whole device
 * (cudaDeviceSynchronize), then copies on the room's own stream, and returns
 * when the copies are complete -- setup calls, never on the step path. */
int rafd_set_state(rafd_room *r, const void *u_prev, const void *u_curr, const void *v, const void *g);

/* Checkpoint / resume: the state of a room is (u^n, u^{n-1}, v, g, step
 * counter n): read it with rafd_read_field / rafd_read_branch_state /
 * rafd_get_info().steps, restore it into a room created from the same inputs
 * with rafd_set_state and rafd_set_step (n indexes the source signal; the
 * boundary copy of u^{n-1} is rebuilt by rafd_set_state).  The continued run
 * is bitwise identical to the uninterrupted one.  STATE on a connected IPC slab. */
int rafd_set_step(rafd_room *r, int64_t n);

/* Enqueue nsteps time steps (volume kernel, boundary kernel, source,
 * receivers, rotation).  Asynchronous w.r.t. the host. */
int rafd_step(rafd_room *r, int64_t nsteps);

/* Temporal blocking: steps_per_sweep = 2 makes
 * rafd_step advance two leapfrog steps per pass over the grid.  The volume
 * update of Listing 2 for step n+2 reads only u^{n+1} on a
 * voxel's 7-point star, so one z-march computes u^{n+1} and, one plane behind,
 * u^{n+2}; the boundary update of step n+1 (Listings 3/4, PAPER.md:371-377,
 * 415-440) and the source then run, and the voxels whose star holds a boundary
 * node or the source (the "shell") get their u^{n+2} recomputed before the
 * boundary update of step n+2.  Results are bitwise those of single steps
 * (same expressions, same order).  Allocates a second pair of field buffers
 * (the two steps are written out of place) and the shell list; an odd step
 * count ends with one single step.  1 switches back (buffers are kept).
 * A z slab (any transport) runs the double step edge planes first: u^{n+1}
 * of its first / last owned plane with the single-step kernel, their exchange
 * overlapped with the two-step kernel over the interior planes, then u^{n+2}
 * of the edge planes from the exchanged u^{n+1}, a second exchange overlapped
 * with the interior shell (one plane per neighbour per step, as single steps).
 * Every slab of a room must use the same setting.  Errors: INVAL (not 1 or
 * 2), STATE (a fused or single-kernel scheme, the v0 kernel, an IPC slab
 * already connected to neighbours that exported two buffers), NOMEM, CUDA. */
int rafd_set_temporal_blocking(rafd_room *r, int32_t steps_per_sweep);

/* Step the n slabs of one room held by this process (created with nranks = n,
 * rank = k, nccl_id = NULL, consecutive [z_begin, z_end)), on one or several
 * devices: per step every slab runs its kernels, then its two ghost planes are
 * copied from its neighbours (cudaMemcpyPeerAsync, event-ordered).  Results
 * are bitwise those of the undivided room.  STATE if the handles are not such
 * a group.  rafd_step on a slab without nccl_id returns STATE. */
int rafd_step_group(rafd_room **rooms, int32_t n, int64_t nsteps);

/* Cross-process slabs without NCCL: a slab created with
 * nranks > 1 and nccl_id = NULL exports a RAFD_IPC_BLOB_BYTES blob (CUDA IPC
 * handles of its field buffers -- two, or four once temporal blocking is on --
 * and of its signal words, plus its plane count and pitch); the caller
 * exchanges blobs (e.g. torch.distributed all_gather_object) and connects each
 * slab to its neighbours' blobs (NULL at the room's ends).  Afterwards
 * rafd_step runs the edge-first step with the halo planes pulled by
 * device-to-device (peer) copies, ordered by GPU-side stream waits on the
 * neighbours' signal words -- no host round trip, no NCCL.  Neighbours may be
 * on the same GPU or on peer GPUs (NVLink).  All slabs must step the same
 * number of times with the same steps_per_sweep; with temporal blocking every
 * slab calls rafd_set_temporal_blocking(r, 2) BEFORE rafd_ipc_handle (the blob
 * then carries the second buffer pair).  Errors: STATE, INVAL, CUDA. */
#define RAFD_IPC_BLOB_BYTES 352
int rafd_ipc_handle(rafd_room *r, uint8_t *blob);
int rafd_ipc_connect(rafd_room *r, const uint8_t *lower, const uint8_t *upper);

/* Device-initiated halo for IPC-connected slabs: instead of
 * pulling the neighbours' edge planes with copies, the kernels that produce a
 * slab's first and last owned planes -- the volume kernel (Listing 2,
 * PAPER.md:349-357) over those planes, the boundary kernel (Listings 3/4,
 * PAPER.md:371-377, 415-440) over their nodes, the source -- also store every
 * value into the neighbour's ghost plane through the peer-mapped buffer, then
 * one GPU-side signal (a stream write with a memory fence) publishes the step.
 * The next step waits for the neighbours' signal of the previous step, which
 * orders both the ghost reads (RAW) and the next pushes (WAR).  Results are
 * bitwise those of the pull transport and of the undivided room.  on = 0
 * selects the pull transport.  Call after rafd_ipc_connect, before the first
 * step; every slab of the room must choose the same transport.  Errors: STATE
 * (not IPC-connected, a fused or single-kernel scheme, the v0 kernel, steps
 * already taken), INVAL. */
int rafd_set_halo_push(rafd_room *r, int32_t on);

/* Wait for all enqueued work of the room. */
int rafd_synchronize(rafd_room *r);

/* All receiver samples recorded since the last read, as double:
 * out[j*cap + k], k < *n_written.  INVAL if cap < number of unread samples. */
int rafd_read_receivers(rafd_room *r, double *out, int64_t cap, int64_t *n_written);

/* u^n (u_curr) and u^{n-1} (u_prev) as T-typed [nz][ny][nx] host or device
 * buffers (the slab's planes for a slab handle).  NULL => skipped. */
int rafd_read_field(rafd_room *r, void *u_curr, void *u_prev);

/* Branch state v, g as T-typed [MB][Nb] host or device buffers. */
int rafd_read_branch_state(rafd_room *r, void *v, void *g);

/* Classification, for bit-exact checks: K [nz][ny][nx] uint8 (0 outside),
 * bidx [Nb] ascending canonical indices of boundary nodes, Kb [Nb], matb [Nb].
 * Host buffers; any may be NULL. */
int rafd_get_classification(rafd_room *r, uint8_t *K, int64_t *bidx, uint8_t *Kb, uint8_t *matb);

int rafd_get_info(rafd_room *r, rafd_info *info);

/* Discrete energy H^{n+1/2} (reading R11) of the current state, accumulated
 * in double on the device (test hook, off the hot path). */
int rafd_energy(rafd_room *r, double *H);

/* Profiling: on != 0 starts accumulating per-kernel times (and resets them). */
int rafd_set_profiling(rafd_room *r, int on);
int rafd_get_kernel_times(rafd_room *r, rafd_kernel_times *t);

/* Number of kernel launches the library has enqueued for this room so far
 * (every launch, including those replayed inside CUDA graphs). */
int64_t rafd_launch_count(rafd_room *r);

/* Host-only helper (no GPU needed): split the nz planes of a room over nranks
 * z-slabs by the prefix sum of the per-plane algorithmic cost
 *   c(z) = 1*N_mask(z) + 3s*N_in(z) + (6 + 3s + 4s*MB)*Nb(z)
 * (SURVEY §8(e)).  mask: host [nz][ny][nx].  Writes z_begin[r], z_end[r]. */
int rafd_slab_plan(int32_t nx, int32_t ny, int32_t nz, const uint8_t *mask, int32_t precision,
                   int32_t n_branches, int32_t nranks, int32_t *z_begin, int32_t *z_end);

/* Device memory.  Whole-room handles (nranks <= 1) take their buffers from a
 * per-device cache owned by the library (a caching allocator over cudaMalloc):
 * rafd_destroy returns them to the cache (which then keeps at most half of the
 * device's memory) instead of freeing them, and the next room of a similar
 * size reuses them.  This call frees every cached block of `device`, e.g.
 * before another library allocates large buffers (like
 * torch.cuda.empty_cache()).  Waits for the device.  Rooms still alive keep
 * their memory.  Also frees the pinned host buffer of the bit-packed mask
 * upload (rafd_create).  INVAL (device < 0), CUDA.  Environment RAFD_POOL=0
 * makes rooms use cudaMalloc / cudaFree directly. */
int rafd_release_cached_memory(int32_t device);

/* 128-byte NCCL unique id for a multi-GPU room (call on rank 0, broadcast). */
int rafd_nccl_unique_id(uint8_t *id128);

const char *rafd_last_error(void);
const char *rafd_strerror(int code);
int rafd_version(void);

#ifdef __cplusplus
}
#endif
#endif /* RAFD_H */
