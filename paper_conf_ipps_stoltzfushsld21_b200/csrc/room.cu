// room.cu -- the C-ABI (include/rafd.h): room lifetime, classification
// orchestration, the per-step launch sequence (row a6: time-level rotation),
// CUDA-graph replay, profiling, and the host-side slab planner.
//
// Per step (Listing 5: volume kernel, then the boundary
// kernel updating the volume in place, "executed iteratively"):
//   k_volume   (u[cur] -> u[cur^1], in place over u^{n-1})
//   k_boundary (nodes of the slab; FI-MM or FD-MM; refreshes ub_prev)
//   k_src_rcv  (soft source + receivers, reading R10)
//   [slab halo exchange over NCCL, multi-GPU only]
//   cur ^= 1
#include <dlfcn.h>
#include <math.h>
#include <stdarg.h>
#include <stdio.h>
#include <stdlib.h>

#include <mutex>
#include <thread>
#include <vector>
#include <string.h>

#include <algorithm>
#include <cfloat>
#include <string>
#include <vector>

#include "internal.cuh"
#include "halo.h"

using namespace rafd;

// ------------------------------------------------------------------ errors
static thread_local std::string g_err;

// Setup-phase tracing (RAFD_TRACE=1): synchronises the room's stream at each
// mark and prints the wall time of the phase to stderr.  Off: one branch.
#include <chrono>
struct PhaseTrace {
    bool on;
    std::chrono::steady_clock::time_point t;
    explicit PhaseTrace(const char *what) : on(getenv("RAFD_TRACE") != nullptr), t(std::chrono::steady_clock::now())
    {
        if (on) fprintf(stderr, "[rafd] %s\n", what);
    }
    void mark(cudaStream_t s, const char *name)
    {
        if (!on) return;
        cudaStreamSynchronize(s);
        const auto n = std::chrono::steady_clock::now();
        fprintf(stderr, "[rafd]   %-28s %8.2f ms\n", name, std::chrono::duration<double, std::milli>(n - t).count());
        t = n;
    }
};

// Work enqueued on a side stream while the main stream does something else
// (setup only): the destructor makes the main stream wait for it, so every
// later use -- and every error path, which synchronises the main stream before
// freeing -- is ordered after it.
struct SideWork {
    cudaStream_t main, side;
    cudaEvent_t ev = nullptr;
    SideWork(cudaStream_t m, cudaStream_t sd) : main(m), side(sd) {}
    void done()
    {
        if (ev) return;
        if (cudaEventCreateWithFlags(&ev, cudaEventDisableTiming) != cudaSuccess || cudaEventRecord(ev, side) != cudaSuccess) {
            cudaStreamSynchronize(side);  // fall back to a host wait
            if (ev) cudaEventDestroy(ev);
            ev = nullptr;
            return;
        }
    }
    ~SideWork()
    {
        if (ev) {
            cudaStreamWaitEvent(main, ev, 0);
            cudaEventDestroy(ev);
        } else {
            cudaStreamSynchronize(side);  // an error path left before done()
        }
    }
};

static int set_err(int code, const char *fmt, ...)
{
    char buf[512];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof buf, fmt, ap);
    va_end(ap);
    g_err = buf;
    return code;
}

#define CK(call)                                                                        \
    do {                                                                                \
        cudaError_t e_ = (call);                                                        \
        if (e_ != cudaSuccess)                                                          \
            return set_err(e_ == cudaErrorMemoryAllocation ? RAFD_E_NOMEM : RAFD_E_CUDA, \
                           "%s: %s (%s:%d)", #call, cudaGetErrorString(e_), __FILE__,   \
                           __LINE__);                                                   \
    } while (0)

static bool is_device_ptr(const void *p)
{
    if (!p) return false;
    cudaPointerAttributes a;
    if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
        cudaGetLastError();
        return false;
    }
    return a.type == cudaMemoryTypeDevice || a.type == cudaMemoryTypeManaged;
}

// A pointer kernels can dereference: device / managed memory as is, pinned
// (page-locked) host memory through its mapped device address (zero-copy over
// PCIe: a kernel then reads exactly the bytes it needs); nullptr for pageable
// host memory (staged through a device buffer instead).
static const void *device_view(const void *p)
{
    if (!p) return nullptr;
    cudaPointerAttributes a;
    if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
        cudaGetLastError();
        return nullptr;
    }
    if (a.type == cudaMemoryTypeDevice || a.type == cudaMemoryTypeManaged) return p;
    if (a.type == cudaMemoryTypeHost && a.devicePointer) return a.devicePointer;
    return nullptr;
}

// ------------------------------------------------------------------ the room
struct rafd_room {
    int device = 0;
    cudaStream_t stream = nullptr, cap_stream = nullptr;
    bool own_stream = false;
    int prec = 32, M = 1, MB = 0;
    size_t s = 4;
    int32_t nx = 0, ny = 0, nz = 0;  // room
    int32_t z0 = 0, z1 = 0;          // owned planes
    int rank = 0, nranks = 1;
    double lambda = 0;
    Grid g{};
    int nsm = 148;
    // field buffers: two pairs.  u[pair + cur] = u^n, u[pair + (cur^1)] =
    // u^{n-1}; a single step writes u^{n+1} in place over u^{n-1} (cur ^= 1), a
    // double step of the two-step kernel (twostep.cu) writes the other pair
    // (pair ^= 2, cur unchanged).  The second pair exists only with temporal
    // blocking on (rafd_set_temporal_blocking).
    void *u[4] = {nullptr, nullptr, nullptr, nullptr};
    int cur = 0;
    int pair = 0;
    int tb = 1;              // steps per HBM sweep (1 or 2)
    void *tbplan = nullptr;  // two-step kernel maps + shell list
    int64_t n_shell = 0;
    uint8_t *K = nullptr, *K_alloc = nullptr;
    int64_t nb = 0;
    bool idx64 = false;
    void *bpos = nullptr;
    int64_t *bidx = nullptr;
    uint8_t *Kb = nullptr, *matb = nullptr;
    void *ub = nullptr, *gst = nullptr, *vst = nullptr;
    void *tab = nullptr;   // T: beta[M] | BI | D | DI | F  ([M*MB] each)
    std::vector<unsigned char> tab_host;  // the same table on the host (boundary-kernel launch parameter)
    bool use_pool = false;                // buffers through the library's memory cache (whole rooms)
    bool shell_bnd = false;               // double steps fuse the shell with the step-(n+2) boundary pass
    double *DF = nullptr;  // double D | F for the energy hook
    void *ctl = nullptr;   // Ctl<T>
    unsigned int *ticket = nullptr;  // last-block ticket of the boundary kernel's fused source/receivers
    void *sig = nullptr;
    int64_t *rcv_pos = nullptr;
    void *rec = nullptr;
    int64_t rec_cap = 0, rec_count = 0;
    void *rec_host = nullptr;  // pinned staging for rafd_read_receivers
    size_t rec_host_bytes = 0;
    int32_t nrcv = 0;
    int64_t steps = 0;
    int64_t k_hist[7] = {0};
    int64_t isolated = 0, n_inside = 0;
    int64_t device_bytes = 0;
    int64_t launches = 0;
    // CUDA graphs of G steps, one per starting parity
    static const int G = 16;
    cudaGraphExec_t graph[4] = {nullptr, nullptr, nullptr, nullptr};  // index pair + cur
    int graph_kernels = 0;
    // profiling
    bool profiling = false;
    struct Ev {
        int kind;
        cudaEvent_t a, b;
    };
    std::vector<Ev> evs;
    std::vector<cudaEvent_t> ev_pool;
    KernelTimes kt;
    // multi-GPU halo exchange: NCCL (one rank per process) or, for slabs of one
    // process (rafd_step_group), device-to-device / peer copies
    Halo *halo = nullptr;
    bool local_slab = false;
    HaloIpc *ipc = nullptr;   // cross-process slabs (rafd_ipc_connect)
    bool push = false;        // IPC halo pushed by the edge-phase kernels (rafd_set_halo_push)
    int64_t *ipc_sig = nullptr;  // [2] IPC signal words (edge done, pulls done)
    // edge-first step of a slab: edge planes, then the halo exchange on
    // comm_stream overlapped with the interior planes
    cudaStream_t comm_stream = nullptr;
    cudaEvent_t ev_edge = nullptr, ev_halo = nullptr;
    int64_t n_first_plane = 0, n_last_start = 0;  // node ranges [0, n_first_plane), [n_last_start, nb)
    int src_z = -1;                                // global plane of the source (-1: none)
    // TMA tensor maps etc. of the volume kernel (nullptr => v0 kernel)
    void *vplan = nullptr;
    bool fused = false;  // boundary update fused into the volume kernel
    int scheme = 0;      // RAFD_SCHEME_*
    double beta1 = 0, loss1 = 1, loss2 = 1;
};

template <typename T> static Ctl<T> *ctl_of(rafd_room *r) { return (Ctl<T> *)r->ctl; }
// the u_b slot of a step whose u^n is u[cur] (null when the boundary update is
// fused into the volume kernel or a single-kernel scheme runs: no ring then)
template <typename T> static T *ub_slot(rafd_room *r, int cur)
{
    return (r->fused || r->scheme || r->nb == 0) ? nullptr : (T *)r->ub + (int64_t)cur * r->nb;
}

template <typename T> static FusedArgs<T> fused_args(const rafd_room *r)
{
    FusedArgs<T> f{};
    f.matb = r->matb;
    f.g = (T *)r->gst;
    f.v = (T *)r->vst;
    f.tab = (const T *)r->tab;
    f.M = r->M;
    f.MB = r->MB;
    f.Nb = r->nb;
    f.l = (T)r->lambda;
    f.scheme = r->scheme;
    f.beta1 = (T)r->beta1;
    f.loss1 = (T)r->loss1;
    f.loss2 = (T)r->loss2;
    return f;
}

// ------------------------------------------------------------------ device memory
// Whole-room handles allocate through the library's cache (devmem.cu); slab
// handles (nranks > 1) with plain cudaMalloc, since their field buffers may be
// exported with CUDA IPC.
// every allocation carries 64 bytes of slack (vector loads / memsets of +16)
static int dmalloc(rafd_room *r, void **p, size_t bytes)
{
    bytes += 64;
    cudaError_t e = dev_alloc(p, bytes, r->use_pool);
    if (e != cudaSuccess) {
        cudaGetLastError();
        *p = nullptr;
        return set_err(RAFD_E_NOMEM, "cudaMalloc(%zu bytes): %s", bytes, cudaGetErrorString(e));
    }
    r->device_bytes += (int64_t)bytes;
    return RAFD_OK;
}

// frees what dmalloc or cudaMalloc returned, once the room's work is done
static void dfree(rafd_room *r, void *p)
{
    if (!p) return;
    cudaStreamSynchronize(r->stream);
    dev_free(p);
}

// ------------------------------------------------------------------ validation
static int validate(const rafd_room_desc *d)
{
    if (!d) return set_err(RAFD_E_INVAL, "null descriptor");
    if (!d->mask) return set_err(RAFD_E_INVAL, "null mask");
    if (d->nx < 1 || d->ny < 1 || d->nz < 1) return set_err(RAFD_E_INVAL, "dims must be >= 1");
    if (d->precision != 32 && d->precision != 64) return set_err(RAFD_E_INVAL, "precision must be 32 or 64");
    if (!d->mat) return set_err(RAFD_E_INVAL, "null materials");
    const rafd_materials *m = d->mat;
    if (m->n_materials < 1 || m->n_materials > RAFD_MAX_MATERIALS) return set_err(RAFD_E_INVAL, "n_materials must be in 1..256");
    if (m->n_branches < 0 || m->n_branches > RAFD_MAX_BRANCHES) return set_err(RAFD_E_INVAL, "n_branches must be in 0..8");
    if (!m->beta0) return set_err(RAFD_E_INVAL, "beta0 is required");
    if (m->n_branches > 0 && (!m->D || !m->E || !m->F)) return set_err(RAFD_E_INVAL, "D, E, F are required when n_branches > 0");
    // reading R1
    if (!(d->lambda > 0.0) || !std::isfinite(d->lambda)) return set_err(RAFD_E_UNSTABLE, "lambda must be finite and > 0");
    if (d->lambda * d->lambda > (1.0 / 3.0) * (1.0 + 4.0 * DBL_EPSILON)) return set_err(RAFD_E_UNSTABLE, "lambda^2 > 1/3");
    // reading R5: passivity
    const int M = m->n_materials, MB = m->n_branches;
    for (int i = 0; i < M; i++) {
        if (!(m->beta0[i] >= 0.0) || !std::isfinite(m->beta0[i])) return set_err(RAFD_E_NONPASSIVE, "beta0[%d] must be finite and >= 0", i);
        for (int b = 0; b < MB; b++) {
            const double D = m->D[i * MB + b], E = m->E[i * MB + b], F = m->F[i * MB + b];
            if (!(D >= 0.0 && E >= 0.0 && F >= 0.0) || !std::isfinite(D) || !std::isfinite(E) || !std::isfinite(F))
                return set_err(RAFD_E_NONPASSIVE, "D, E, F of material %d branch %d must be finite and >= 0", i, b);
        }
    }
    if (d->scheme < 0 || d->scheme > 2) return set_err(RAFD_E_INVAL, "scheme must be 0, 1 or 2");
    if (d->scheme == 1 && (m->n_materials != 1 || m->n_branches != 0))
        return set_err(RAFD_E_INVAL, "Listing 1 has one admittance: n_materials = 1 and n_branches = 0");
    if (d->scheme == 2 && (m->n_branches != 0 || !std::isfinite(d->loss1) || !std::isfinite(d->loss2)))
        return set_err(RAFD_E_INVAL, "Listing 6 needs n_branches = 0 and finite loss1, loss2");
    if (d->mask_z0 < 0 || d->mask_z0 > std::max(0, (d->nranks > 1 ? d->z_begin : 0) - 1))
        return set_err(RAFD_E_INVAL, "mask_z0 must be <= the first plane read (z_begin-1, clipped)");
    if (d->nranks > 1) {
        if (d->rank < 0 || d->rank >= d->nranks) return set_err(RAFD_E_INVAL, "rank out of range");
        if (!(d->z_begin >= 0 && d->z_begin < d->z_end && d->z_end <= d->nz))
            return set_err(RAFD_E_INVAL, "slab [z_begin, z_end) must be a non-empty range of planes (use rafd_slab_plan)");
    }
    return RAFD_OK;
}

// Derived per-material coefficients (reading R5), in double, then rounded to T.
template <typename T>
static void build_tables(const rafd_materials *m, std::vector<T> &tab, std::vector<double> &DF)
{
    const int M = m->n_materials, MB = m->n_branches;
    tab.assign((size_t)M * (1 + 4 * MB), (T)0);
    DF.assign((size_t)2 * M * MB + 1, 0.0);
    T *beta = tab.data(), *BI = beta + M, *D = BI + M * MB, *DI = D + M * MB, *F = DI + M * MB;
    for (int i = 0; i < M; i++) {
        double bsum = m->beta0[i];
        for (int b = 0; b < MB; b++) {
            const int k = i * MB + b;
            const double d = m->D[k], e = m->E[k], f = m->F[k];
            const bool unused = (d == 0.0 && e == 0.0 && f == 0.0);
            const double bi = unused ? 0.0 : 1.0 / ((2.0 * d + e) + f);
            const double di = (2.0 * d - e) - f;
            bsum = bsum + bi;
            BI[k] = (T)bi;
            D[k] = (T)d;
            DI[k] = (T)di;
            F[k] = (T)f;
            DF[k] = d;
            DF[(size_t)M * MB + k] = f;
        }
        beta[i] = (T)bsum;
    }
}

// Copy nplanes planes (each plane_bytes) starting at plane zg0 of a host or
// device array into `staging` chunk by chunk and call fn(chunk_ptr, zg, n).
// `src` holds planes [src_z0, ...) of the room.
template <typename Fn>
static int for_plane_chunks(rafd_room *r, const void *src, int src_z0, bool dev, size_t plane_bytes,
                            int zg0, int nplanes, void *staging, size_t staging_bytes, Fn fn)
{
    if (nplanes <= 0) return RAFD_OK;
    if (dev) return fn((const char *)src + (size_t)(zg0 - src_z0) * plane_bytes, zg0, nplanes);
    int per = (int)std::max<size_t>(1, staging_bytes / plane_bytes);
    for (int z = zg0; z < zg0 + nplanes; z += per) {
        const int n = std::min(per, zg0 + nplanes - z);
        CK(cudaMemcpyAsync(staging, (const char *)src + (size_t)(z - src_z0) * plane_bytes, (size_t)n * plane_bytes,
                           cudaMemcpyHostToDevice, r->stream));
        int rc = fn(staging, z, n);
        if (rc) return rc;
        CK(cudaStreamSynchronize(r->stream));  // staging reused by the next chunk
    }
    return RAFD_OK;
}

static const size_t kStagingBytes = 256ull << 20;

// Bit-packed upload of a host mask (maskpack.cu, classify.cu k_scatter_mask_bits):
// the classification needs one bit per voxel, the mask has a byte (C4: the
// 1.1 GB byte mask crossed PCIe in 20.4 ms).  Host threads each pack a range of
// planes into a pinned buffer and issue its copy as soon as it is packed, so the
// 1/8-size copies overlap the packing; the device expands the bits into K.
// Rounds of at most kStagingBytes packed.  The pinned buffer is shared by the
// process's rooms (grown on demand).  RAFD_MASK_BITS=0 keeps the byte stream.
// Returns -1 when not applicable (the caller then streams bytes).
static std::mutex g_pack_mu;
static void *g_pack_host = nullptr;
static size_t g_pack_bytes = 0;

static int upload_mask_bits(rafd_room *r, const uint8_t *mask, int mz0, int zg0, int nplanes, void *staging)
{
    if (const char *e = getenv("RAFD_MASK_BITS"))
        if (atoi(e) == 0) return -1;
    const Grid &g = r->g;
    const int rw = (r->nx + 31) / 32;
    const size_t plane_b = (size_t)r->ny * rw * 4, nxny = (size_t)r->nx * r->ny;
    if (nplanes <= 0 || plane_b > kStagingBytes) return -1;
    const int per_round = (int)std::min<size_t>((size_t)nplanes, kStagingBytes / plane_b);
    std::lock_guard<std::mutex> lk(g_pack_mu);
    const size_t need = (size_t)per_round * plane_b;
    if (g_pack_bytes < need) {
        if (g_pack_host) cudaFreeHost(g_pack_host);
        g_pack_host = nullptr;
        g_pack_bytes = 0;
        if (cudaHostAlloc(&g_pack_host, need, cudaHostAllocPortable) != cudaSuccess) {
            cudaGetLastError();
            g_pack_host = nullptr;
            return -1;
        }
        g_pack_bytes = need;
    }
    const int nt = std::max(1, std::min(pack_threads(), per_round));
    std::vector<cudaStream_t> cs(nt, nullptr);
    std::vector<cudaEvent_t> ce(nt, nullptr);
    cudaError_t e = cudaSuccess;
    for (int t = 0; t < nt && e == cudaSuccess; t++) {
        e = cudaStreamCreateWithFlags(&cs[t], cudaStreamNonBlocking);
        if (e == cudaSuccess) e = cudaEventCreateWithFlags(&ce[t], cudaEventDisableTiming);
    }
    for (int z = zg0; z < zg0 + nplanes && e == cudaSuccess; z += per_round) {
        const int n = std::min(per_round, zg0 + nplanes - z);
        // the previous round's expansion has read the device buffer (stream order
        // on r->stream is not enough: the copies run on the packing threads' streams)
        e = cudaStreamSynchronize(r->stream);
        if (e != cudaSuccess) break;
        std::vector<cudaError_t> te(nt, cudaSuccess);
        auto part = [&](int t) {
            const int p0 = (int)((int64_t)n * t / nt), p1 = (int)((int64_t)n * (t + 1) / nt);
            if (p0 >= p1) return;
            cudaSetDevice(r->device);  // a new thread starts on device 0
            uint32_t *hb = (uint32_t *)((char *)g_pack_host + (size_t)p0 * plane_b);
            pack_mask_rows(mask + (size_t)(z + p0 - mz0) * nxny, (int64_t)(p1 - p0) * r->ny, r->nx, hb, rw, 1);
            te[t] = cudaMemcpyAsync((char *)staging + (size_t)p0 * plane_b, hb, (size_t)(p1 - p0) * plane_b,
                                    cudaMemcpyHostToDevice, cs[t]);
            if (te[t] == cudaSuccess) te[t] = cudaEventRecord(ce[t], cs[t]);
        };
        std::vector<std::thread> th;
        th.reserve(nt);
        int spawned = 0;
        try {
            for (int t = 1; t < nt; t++, spawned++) th.emplace_back(part, t);
        } catch (...) {  // no threads to be had: the caller's thread packs the rest
        }
        part(0);
        for (int t = 1 + spawned; t < nt; t++) part(t);
        for (auto &t : th) t.join();
        for (int t = 0; t < nt && e == cudaSuccess; t++) {
            const int p0 = (int)((int64_t)n * t / nt), p1 = (int)((int64_t)n * (t + 1) / nt);
            if (p0 >= p1) continue;
            e = te[t];
            if (e == cudaSuccess) e = cudaStreamWaitEvent(r->stream, ce[t], 0);
        }
        if (e == cudaSuccess)
            e = launch_scatter_mask_bits(g, (const uint32_t *)staging, rw, z - r->z0 + 1, n, r->K, r->stream);
    }
    // the pinned buffer is reused by the next room: drain before unlocking
    const cudaError_t e2 = cudaStreamSynchronize(r->stream);
    if (e == cudaSuccess) e = e2;
    for (int t = 0; t < nt; t++) {
        if (cs[t]) cudaStreamSynchronize(cs[t]), cudaStreamDestroy(cs[t]);
        if (ce[t]) cudaEventDestroy(ce[t]);
    }
    if (e != cudaSuccess) return set_err(RAFD_E_CUDA, "mask upload: %s", cudaGetErrorString(e));
    return RAFD_OK;
}

template <typename T> static int create_t(rafd_room *r, const rafd_room_desc *d)
{
    const int64_t nxny = (int64_t)r->nx * r->ny;
    Grid &g = r->g;
    g.nx = r->nx;
    g.ny = r->ny;
    g.lnz = r->z1 - r->z0;
    g.xo = (int)(128 / sizeof(T));
    const int64_t align = 128 / (int64_t)sizeof(T);
    g.pitch = ((g.xo + r->nx + 1 + align - 1) / align) * align;
    g.plane = g.pitch * (r->ny + 2);
    g.total = g.plane * (g.lnz + 2);
    r->idx64 = g.total >= (int64_t)UINT32_MAX;

    int rc;
    PhaseTrace tr("rafd_create");
    // K grid: element (row, xo + x) must sit at a 16-byte aligned byte address
    // for the TMA boxes of the volume kernel, so the buffer starts k_shift(g)
    // bytes before the first element (r->K_alloc is what cudaMalloc returned).
    if ((rc = dmalloc(r, (void **)&r->K_alloc, (size_t)g.total + 64))) return rc;
    r->K = r->K_alloc + k_shift(g);
    for (int k = 0; k < 2; k++)
        if ((rc = dmalloc(r, &r->u[k], (size_t)g.total * sizeof(T) + 64))) return rc;
    tr.mark(r->stream, "alloc K, u[2]");
    CK(cudaMemsetAsync(r->K_alloc, 0, (size_t)g.total + 64, r->stream));
    // the two field buffers are zeroed on the side stream while the mask streams
    // in over PCIe (C4: 1.5 ms of memset hidden behind the 20 ms H2D); the main
    // stream waits for it when create_t returns
    SideWork zero_u(r->stream, r->cap_stream);
    for (int k = 0; k < 2; k++) CK(cudaMemsetAsync(r->u[k], 0, (size_t)g.total * sizeof(T) + 64, r->cap_stream));
    zero_u.done();
    tr.mark(r->stream, "memset K");

    // ---- classification (row a1)
    // the mask is streamed in full (DMA staging beats zero-copy reads for it);
    // the matmap is only sampled at boundary nodes, so pinned host memory is
    // read in place by the gather kernel
    const void *mask_dv = is_device_ptr(d->mask) ? d->mask : nullptr, *matmap_dv = device_view(d->matmap);
    const bool mdev = mask_dv != nullptr;
    void *staging = nullptr;
    if ((!mdev || (d->matmap && !matmap_dv)) && (rc = dmalloc(r, &staging, kStagingBytes))) return rc;
    const int zlo = std::max(0, r->z0 - 1), zhi = std::min(r->nz, r->z1 + 1);  // incl. ghost planes
    const int mz0 = d->mask_z0;
    rc = mdev ? -1 : upload_mask_bits(r, (const uint8_t *)d->mask, mz0, zlo, zhi - zlo, staging);
    if (rc == -1)
        rc = for_plane_chunks(r, mdev ? mask_dv : d->mask, mz0, mdev, (size_t)nxny, zlo, zhi - zlo, staging,
                              kStagingBytes, [&](const void *chunk, int zg, int n) -> int {
                                  CK(launch_scatter_mask(g, (const uint8_t *)chunk, zg - r->z0 + 1, n, r->K,
                                                         r->stream));
                                  return RAFD_OK;
                              });
    if (rc) return rc;
    tr.mark(r->stream, "mask H2D + scatter");
    CK(launch_count_k(g, r->K, r->stream));
    unsigned long long *hist = nullptr;
    if ((rc = dmalloc(r, (void **)&hist, 8 * sizeof(unsigned long long) + sizeof(unsigned)))) return rc;
    CK(cudaMemsetAsync(hist, 0, 8 * sizeof(unsigned long long) + sizeof(unsigned), r->stream));
    CK(launch_finish_k(g, r->K, hist, r->stream));
    const int64_t rows = (int64_t)g.lnz * r->ny;
    int64_t *counts = nullptr, *row_off = nullptr;
    if ((rc = dmalloc(r, (void **)&counts, (size_t)(rows + 1) * 8))) return rc;
    if ((rc = dmalloc(r, (void **)&row_off, (size_t)(rows + 1) * 8))) return rc;
    CK(cudaMemsetAsync(counts, 0, (size_t)(rows + 1) * 8, r->stream));
    CK(launch_row_counts64(g, r->K, counts, r->stream));
    size_t tmpb = 0;
    CK(exclusive_scan_rows64(counts, row_off, rows + 1, nullptr, &tmpb, r->stream));
    void *tmp = nullptr;
    if ((rc = dmalloc(r, &tmp, tmpb))) return rc;
    CK(exclusive_scan_rows64(counts, row_off, rows + 1, tmp, &tmpb, r->stream));
    unsigned long long h[8];
    CK(cudaMemcpyAsync(h, hist, sizeof h, cudaMemcpyDeviceToHost, r->stream));
    CK(cudaMemcpyAsync(&r->nb, row_off + rows, 8, cudaMemcpyDeviceToHost, r->stream));
    // boundary nodes of the first / last owned plane (edge phase of a slab)
    CK(cudaMemcpyAsync(&r->n_first_plane, row_off + std::min<int64_t>(rows, r->ny), 8, cudaMemcpyDeviceToHost, r->stream));
    CK(cudaMemcpyAsync(&r->n_last_start, row_off + (int64_t)(g.lnz - 1) * r->ny, 8, cudaMemcpyDeviceToHost, r->stream));
    CK(cudaStreamSynchronize(r->stream));
    tr.mark(r->stream, "K, histogram, row scan");
    r->isolated = (int64_t)h[0];
    int64_t nin = 0;
    for (int k = 1; k <= 6; k++) {
        r->k_hist[k] = (int64_t)h[k];
        nin += (int64_t)h[k];
    }
    r->n_inside = nin;
    r->k_hist[0] = (int64_t)g.lnz * nxny - nin;

    const int64_t nb = r->nb;
    if ((rc = dmalloc(r, &r->bpos, (size_t)nb * (r->idx64 ? 8 : 4)))) return rc;
    if ((rc = dmalloc(r, (void **)&r->bidx, (size_t)nb * 8))) return rc;
    if ((rc = dmalloc(r, (void **)&r->Kb, (size_t)nb))) return rc;
    if ((rc = dmalloc(r, (void **)&r->matb, (size_t)nb))) return rc;
    if ((rc = dmalloc(r, &r->ub, (size_t)2 * nb * sizeof(T)))) return rc;  // [2][Nb] ring, slot = cur
    if ((rc = dmalloc(r, &r->gst, (size_t)nb * r->MB * sizeof(T)))) return rc;
    if ((rc = dmalloc(r, &r->vst, (size_t)nb * r->MB * sizeof(T)))) return rc;
    CK(cudaMemsetAsync(r->ub, 0, (size_t)2 * nb * sizeof(T) + 16, r->stream));
    CK(cudaMemsetAsync(r->gst, 0, (size_t)nb * r->MB * sizeof(T) + 16, r->stream));
    CK(cudaMemsetAsync(r->vst, 0, (size_t)nb * r->MB * sizeof(T) + 16, r->stream));
    CK(launch_compact(g, r->K, row_off, r->z0, r->ny, r->nx, r->idx64, r->bpos, r->bidx, r->Kb, r->stream));
    tr.mark(r->stream, "boundary SoA alloc + compact");

    // material ids at the boundary nodes (reading R4)
    unsigned *bad = (unsigned *)(hist + 8);
    if (!d->matmap) {
        CK(cudaMemsetAsync(r->matb, 0, (size_t)nb + 1, r->stream));
    } else if (matmap_dv) {  // device memory, or pinned host memory read in place
        CK(launch_gather_mat((const uint8_t *)matmap_dv, (int64_t)mz0 * nxny, r->bidx, 0, nb, r->matb, r->M, bad,
                             r->stream));
    } else {
        std::vector<int64_t> off_h((size_t)rows + 1);
        CK(cudaMemcpyAsync(off_h.data(), row_off, (size_t)(rows + 1) * 8, cudaMemcpyDeviceToHost, r->stream));
        CK(cudaStreamSynchronize(r->stream));
        rc = for_plane_chunks(r, d->matmap, mz0, false, (size_t)nxny, r->z0, g.lnz, staging, kStagingBytes,
                              [&](const void *chunk, int zg, int n) -> int {
                                  const int64_t i_lo = off_h[(size_t)(zg - r->z0) * r->ny];
                                  const int64_t i_hi = off_h[(size_t)(zg - r->z0 + n) * r->ny];
                                  CK(launch_gather_mat((const uint8_t *)chunk, (int64_t)zg * nxny, r->bidx,
                                                       i_lo, i_hi, r->matb, r->M, bad, r->stream));
                                  return RAFD_OK;
                              });
        if (rc) return rc;
    }
    unsigned bad_h = 0;
    tr.mark(r->stream, "material gather");
    CK(cudaMemcpyAsync(&bad_h, bad, sizeof bad_h, cudaMemcpyDeviceToHost, r->stream));
    CK(cudaStreamSynchronize(r->stream));
    dfree(r, hist);
    dfree(r, counts);
    dfree(r, row_off);
    dfree(r, tmp);
    dfree(r, staging);
    r->device_bytes -= (int64_t)(8 * sizeof(unsigned long long) + sizeof(unsigned)) + 2 * (rows + 1) * 8 +
                       (int64_t)(tmpb ? tmpb : 16) + (staging ? (int64_t)kStagingBytes : 0);
    if (bad_h) return set_err(RAFD_E_MATERIAL, "matmap holds a material id >= n_materials (%d) at a boundary node", r->M);

    // ---- tables, control block
    std::vector<T> tab;
    std::vector<double> DF;
    build_tables<T>(d->mat, tab, DF);
    if ((rc = dmalloc(r, &r->tab, tab.size() * sizeof(T)))) return rc;
    if ((rc = dmalloc(r, (void **)&r->DF, DF.size() * sizeof(double)))) return rc;
    CK(cudaMemcpy(r->tab, tab.data(), tab.size() * sizeof(T), cudaMemcpyHostToDevice));
    r->tab_host.assign((const unsigned char *)tab.data(), (const unsigned char *)(tab.data() + tab.size()));
    CK(cudaMemcpy(r->DF, DF.data(), DF.size() * sizeof(double), cudaMemcpyHostToDevice));
    if ((rc = dmalloc(r, &r->ctl, sizeof(Ctl<T>)))) return rc;
    if ((rc = dmalloc(r, (void **)&r->ticket, sizeof(unsigned int)))) return rc;
    CK(cudaMemset(r->ticket, 0, sizeof(unsigned int)));
    Ctl<T> c{};
    c.src_pos = -1;
    c.src_node = -1;
    CK(cudaMemcpy(r->ctl, &c, sizeof c, cudaMemcpyHostToDevice));
    tr.mark(r->stream, "tables, control block");
    const char *env = getenv("RAFD_VOLUME_KERNEL");
    if (!(env && strcmp(env, "v0") == 0)) {
        CK(volume_plan_create<T>(g, r->u, r->K_alloc, r->nsm, &r->vplan));
        tr.mark(r->stream, "volume plan: maps, attributes");
        const char *sk = getenv("RAFD_SKIP_EMPTY");  // skipping of all-outside tile-planes (default on)
        if (!(sk && strcmp(sk, "0") == 0)) CK(volume_plan_occupancy(r->vplan, g, r->K, r->stream));
    }
    tr.mark(r->stream, "volume plan: occupancy");
    // boundary update fused into the volume kernel with RAFD_FUSED=1 (DESIGN.md
    // §6; needs the default tiling, MB <= 4, Nb < 2^31).  Off by default: the
    // first fused form is latency-bound at x-wall rows (5.6 ms vs 2.55 ms).
    const char *fz = getenv("RAFD_FUSED");
    if (r->vplan && fz && strcmp(fz, "1") == 0 && r->MB <= 4 && nb < INT32_MAX && r->scheme == 0) {
        cudaError_t e = volume_plan_fuse(r->vplan, g, r->K, nb, r->stream);
        if (e != cudaSuccess && e != cudaErrorNotSupported) CK(e);
        cudaGetLastError();
        r->fused = volume_plan_fused(r->vplan);
    }
    return RAFD_OK;
}

extern "C" int rafd_create(const rafd_room_desc *d, rafd_room **out)
{
    if (!out) return set_err(RAFD_E_INVAL, "null out");
    *out = nullptr;
    int rc = validate(d);
    if (rc) return rc;
    int ndev = 0;
    if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0) {
        cudaGetLastError();
        return set_err(RAFD_E_CUDA, "no CUDA device (there is no CPU fallback)");
    }
    if (d->device < 0 || d->device >= ndev) return set_err(RAFD_E_INVAL, "device %d out of range", d->device);
    CK(cudaSetDevice(d->device));
    // device inputs may still be in flight on any of the caller's streams: the
    // room's stream is non-blocking, so wait for the device first (setup call)
    if (is_device_ptr(d->mask) || (d->matmap && is_device_ptr(d->matmap))) CK(cudaDeviceSynchronize());
    // L2 fetch granularity (experiment knob; device-wide, so opt-in only)
    if (const char *lf = getenv("RAFD_L2_FETCH")) cudaDeviceSetLimit(cudaLimitMaxL2FetchGranularity, (size_t)atoi(lf));
    rafd_room *r = new rafd_room();
    r->device = d->device;
    r->prec = d->precision;
    r->s = d->precision == 32 ? 4 : 8;
    r->M = d->mat->n_materials;
    r->MB = d->mat->n_branches;
    r->nx = d->nx;
    r->ny = d->ny;
    r->nz = d->nz;
    r->lambda = d->lambda;
    r->scheme = d->scheme;
    r->beta1 = d->mat->beta0[0];
    r->loss1 = d->loss1;
    r->loss2 = d->loss2;
    r->rank = d->nranks > 1 ? d->rank : 0;
    r->nranks = d->nranks > 1 ? d->nranks : 1;
    r->z0 = r->nranks > 1 ? d->z_begin : 0;
    r->z1 = r->nranks > 1 ? d->z_end : d->nz;
    r->use_pool = r->nranks == 1 && dev_cache_enabled();
    cudaDeviceGetAttribute(&r->nsm, cudaDevAttrMultiProcessorCount, r->device);
    if (d->cuda_stream) {
        r->stream = (cudaStream_t)d->cuda_stream;
    } else {
        cudaError_t e = cudaStreamCreateWithFlags(&r->stream, cudaStreamNonBlocking);
        if (e != cudaSuccess) {
            delete r;
            return set_err(RAFD_E_CUDA, "cudaStreamCreate: %s", cudaGetErrorString(e));
        }
        r->own_stream = true;
    }
    cudaStreamCreateWithFlags(&r->cap_stream, cudaStreamNonBlocking);
    rc = r->prec == 32 ? create_t<float>(r, d) : create_t<double>(r, d);
    if (!rc && r->nranks > 1) {
        if (d->nccl_id) {
            rc = halo_create(&r->halo, d->nccl_id, r->rank, r->nranks, r->stream);
            if (rc) set_err(rc, "%s", halo_last_error());
        } else {
            r->local_slab = true;  // stepped by rafd_step_group in this process
        }
        cudaStreamCreateWithFlags(&r->comm_stream, cudaStreamNonBlocking);
        if (!rc && cudaMalloc((void **)&r->ipc_sig, 64) == cudaSuccess) cudaMemset(r->ipc_sig, 0, 64);
        cudaEventCreateWithFlags(&r->ev_edge, cudaEventDisableTiming);
        cudaEventCreateWithFlags(&r->ev_halo, cudaEventDisableTiming);
    }
    if (rc) {
        std::string keep = g_err;
        rafd_destroy(r);
        g_err = keep;
        return rc;
    }
    *out = r;
    return RAFD_OK;
}

static void free_graphs(rafd_room *r)
{
    for (int p = 0; p < 4; p++)
        if (r->graph[p]) {
            cudaGraphExecDestroy(r->graph[p]);
            r->graph[p] = nullptr;
        }
}

extern "C" void rafd_destroy(rafd_room *r)
{
    if (!r) return;
    cudaSetDevice(r->device);
    if (r->stream) cudaStreamSynchronize(r->stream);
    PhaseTrace tr("rafd_destroy");
    free_graphs(r);
    if (r->halo) halo_destroy(r->halo);
    if (r->ipc) ipc_close(r->ipc);
    if (r->ipc_sig) cudaFree(r->ipc_sig);
    if (r->ev_edge) cudaEventDestroy(r->ev_edge);
    if (r->ev_halo) cudaEventDestroy(r->ev_halo);
    if (r->comm_stream) cudaStreamDestroy(r->comm_stream);
    if (r->vplan) volume_plan_destroy(r->vplan);
    if (r->tbplan) twostep_plan_destroy(r->tbplan);
    void *ps[] = {r->u[0], r->u[1], r->u[2], r->u[3], r->K_alloc, r->bpos, r->bidx, r->Kb, r->matb, r->ub, r->gst, r->vst,
                  r->tab, r->DF, r->ctl, r->ticket, r->sig, r->rcv_pos, r->rec};
    for (void *p : ps) dfree(r, p);
    tr.mark(r->stream, "free device buffers");
    for (auto &e : r->evs) {
        cudaEventDestroy(e.a);
        cudaEventDestroy(e.b);
    }
    for (auto e : r->ev_pool) cudaEventDestroy(e);
    if (r->rec_host) cudaFreeHost(r->rec_host);
    if (r->cap_stream) cudaStreamDestroy(r->cap_stream);
    if (r->own_stream && r->stream) cudaStreamDestroy(r->stream);
    if (r->use_pool) {  // keep at most half of the device memory cached
        size_t fr = 0, tot = 0;
        if (cudaMemGetInfo(&fr, &tot) == cudaSuccess) dev_cache_trim(r->device, tot / 2);
    }
    cudaGetLastError();
    delete r;
}

extern "C" int rafd_release_cached_memory(int32_t device)
{
    if (device < 0) return set_err(RAFD_E_INVAL, "device must be >= 0");
    CK(cudaSetDevice(device));
    CK(cudaDeviceSynchronize());
    dev_cache_trim(device, 0);
    {  // the pinned staging of the bit-packed mask upload (process-wide)
        std::lock_guard<std::mutex> lk(g_pack_mu);
        if (g_pack_host) cudaFreeHost(g_pack_host);
        g_pack_host = nullptr;
        g_pack_bytes = 0;
    }
    return RAFD_OK;
}

// ------------------------------------------------------------------ source / receivers
static bool owns_plane(const rafd_room *r, int z) { return z >= r->z0 && z < r->z1; }

static int64_t pad_pos(const rafd_room *r, int x, int y, int z)
{
    return (int64_t)(z - r->z0 + 1) * r->g.plane + (int64_t)(y + 1) * r->g.pitch + r->g.xo + x;
}

static int k_at(rafd_room *r, int64_t p, uint8_t *k)
{
    CK(cudaStreamSynchronize(r->stream));
    CK(cudaMemcpy(k, r->K + p, 1, cudaMemcpyDeviceToHost));
    return RAFD_OK;
}

template <typename T> static int push_ctl(rafd_room *r, const Ctl<T> &c)
{
    CK(cudaStreamSynchronize(r->stream));
    CK(cudaMemcpy(r->ctl, &c, sizeof c, cudaMemcpyHostToDevice));
    return RAFD_OK;
}

template <typename T> static int pull_ctl(rafd_room *r, Ctl<T> &c)
{
    CK(cudaStreamSynchronize(r->stream));
    CK(cudaMemcpy(&c, r->ctl, sizeof c, cudaMemcpyDeviceToHost));
    return RAFD_OK;
}

template <typename T>
static int set_source_t(rafd_room *r, int32_t x, int32_t y, int32_t z, const double *sig, int64_t len)
{
    Ctl<T> c;
    int rc = pull_ctl<T>(r, c);
    if (rc) return rc;
    if (r->sig) {
        cudaFree(r->sig);
        r->sig = nullptr;
    }
    c.sig = nullptr;
    c.sig_len = 0;
    c.src_pos = -1;
    c.src_node = -1;
    r->src_z = -1;
    if (len > 0 && owns_plane(r, z)) {
        const int64_t p = pad_pos(r, x, y, z);
        uint8_t k = 0;
        if ((rc = k_at(r, p, &k))) return rc;
        if (k == 0) return set_err(RAFD_E_OUTSIDE, "source (%d,%d,%d) is at an outside voxel", x, y, z);
        std::vector<T> st((size_t)len);
        for (int64_t i = 0; i < len; i++) st[(size_t)i] = (T)sig[i];
        CK(cudaMalloc(&r->sig, (size_t)len * sizeof(T)));
        CK(cudaMemcpy(r->sig, st.data(), (size_t)len * sizeof(T), cudaMemcpyHostToDevice));
        c.sig = (const T *)r->sig;
        c.sig_len = len;
        c.src_pos = p;
        if (k < 6 && r->nb > 0) {  // a boundary node: its u_b slot follows the source too
            int64_t *dn = nullptr;
            CK(cudaMalloc(&dn, 8));
            cudaError_t e = launch_find_node(r->bpos, r->idx64, r->nb, p, dn, r->stream);
            if (e == cudaSuccess) e = cudaMemcpyAsync(&c.src_node, dn, 8, cudaMemcpyDeviceToHost, r->stream);
            if (e == cudaSuccess) e = cudaStreamSynchronize(r->stream);
            cudaFree(dn);
            CK(e);
        }
        r->src_z = z;
    }
    // temporal blocking: the source's 7-point star is recomputed with the shell
    if (r->tbplan) CK(twostep_set_source(r->tbplan, c.src_pos, r->g));
    return push_ctl<T>(r, c);
}

extern "C" int rafd_set_source(rafd_room *r, int32_t x, int32_t y, int32_t z, const double *sig, int64_t len)
{
    if (!r || len < 0 || (len > 0 && !sig)) return set_err(RAFD_E_INVAL, "bad source arguments");
    if (x < 0 || y < 0 || z < 0 || x >= r->nx || y >= r->ny || z >= r->nz)
        return set_err(RAFD_E_OUTSIDE, "source (%d,%d,%d) outside the grid", x, y, z);
    CK(cudaSetDevice(r->device));
    return r->prec == 32 ? set_source_t<float>(r, x, y, z, sig, len) : set_source_t<double>(r, x, y, z, sig, len);
}

template <typename T> static int set_receivers_t(rafd_room *r, int32_t n, const int32_t *xyz)
{
    std::vector<int64_t> pos((size_t)n);
    for (int j = 0; j < n; j++) {
        const int x = xyz[3 * j], y = xyz[3 * j + 1], z = xyz[3 * j + 2];
        if (x < 0 || y < 0 || z < 0 || x >= r->nx || y >= r->ny || z >= r->nz)
            return set_err(RAFD_E_OUTSIDE, "receiver %d (%d,%d,%d) outside the grid", j, x, y, z);
        if (!owns_plane(r, z)) {
            pos[(size_t)j] = 0;  // padded element 0 is a halo corner: always +0
            continue;
        }
        pos[(size_t)j] = pad_pos(r, x, y, z);
        uint8_t k = 0;
        int rc = k_at(r, pos[(size_t)j], &k);
        if (rc) return rc;
        if (k == 0) return set_err(RAFD_E_OUTSIDE, "receiver %d (%d,%d,%d) is at an outside voxel", j, x, y, z);
    }
    Ctl<T> c;
    int rc = pull_ctl<T>(r, c);
    if (rc) return rc;
    if (r->rcv_pos) cudaFree(r->rcv_pos);
    if (r->rec) cudaFree(r->rec);
    r->rcv_pos = nullptr;
    r->rec = nullptr;
    r->rec_cap = r->rec_count = 0;
    r->nrcv = n;
    if (n > 0) {
        CK(cudaMalloc((void **)&r->rcv_pos, (size_t)n * 8));
        CK(cudaMemcpy(r->rcv_pos, pos.data(), (size_t)n * 8, cudaMemcpyHostToDevice));
    }
    c.rcv_pos = r->rcv_pos;
    c.nrcv = n;
    c.rec = nullptr;
    c.rec_cap = 0;
    c.rec_count = 0;
    return push_ctl<T>(r, c);
}

extern "C" int rafd_set_receivers(rafd_room *r, int32_t n, const int32_t *xyz)
{
    if (!r || n < 0 || (n > 0 && !xyz)) return set_err(RAFD_E_INVAL, "bad receiver arguments");
    CK(cudaSetDevice(r->device));
    return r->prec == 32 ? set_receivers_t<float>(r, n, xyz) : set_receivers_t<double>(r, n, xyz);
}

// grow the receiver buffer so that `more` further steps fit
template <typename T> static int ensure_rec(rafd_room *r, int64_t more)
{
    if (r->nrcv == 0 || r->rec_count + more <= r->rec_cap) return RAFD_OK;
    int64_t cap = std::max<int64_t>(1024, r->rec_cap * 2);
    while (cap < r->rec_count + more) cap *= 2;
    void *nb = nullptr;
    CK(cudaStreamSynchronize(r->stream));
    CK(cudaMalloc(&nb, (size_t)cap * r->nrcv * sizeof(T)));
    if (r->rec && r->rec_count)
        CK(cudaMemcpy(nb, r->rec, (size_t)r->rec_count * r->nrcv * sizeof(T), cudaMemcpyDeviceToDevice));
    if (r->rec) cudaFree(r->rec);
    r->rec = nb;
    r->rec_cap = cap;
    Ctl<T> c;
    int rc = pull_ctl<T>(r, c);
    if (rc) return rc;
    c.rec = (T *)nb;
    c.rec_cap = cap;
    return push_ctl<T>(r, c);
}

// ------------------------------------------------------------------ stepping
// the profiling wrapper: CUDA events around one launch on stream s
template <typename Fn> static cudaError_t timed_launch(rafd_room *r, cudaStream_t s, bool prof, int kind, Fn fn)
{
    if (!prof) return fn();
    cudaEvent_t a, b;
    if (r->ev_pool.size() >= 2) {
        a = r->ev_pool.back();
        r->ev_pool.pop_back();
        b = r->ev_pool.back();
        r->ev_pool.pop_back();
    } else {
        cudaEventCreate(&a);
        cudaEventCreate(&b);
    }
    cudaEventRecord(a, s);
    cudaError_t e = fn();
    cudaEventRecord(b, s);
    r->evs.push_back({kind, a, b});
    return e;
}

// one step from the state (pair, cur): u^n = u[pair+cur] -> u^{n+1} in place over u[pair+(cur^1)]
template <typename T> static cudaError_t enqueue_step(rafd_room *r, int pair, int cur, cudaStream_t s, bool prof)
{
    const Grid &g = r->g;
    T *uc = (T *)r->u[pair + cur];
    T *un = (T *)r->u[pair + (cur ^ 1)];
    auto timed = [&](int kind, auto fn) -> cudaError_t { return timed_launch(r, s, prof, kind, fn); };
    const FusedArgs<T> fa = fused_args<T>(r);
    cudaError_t e = timed(0, [&] {
        return launch_volume<T>(g, uc, un, r->K, r->lambda, 0, g.lnz, s, r->vplan, pair + cur,
                                (r->fused || r->scheme) ? &fa : nullptr);
    });
    if (e != cudaSuccess) return e;
    if (r->nb > 0 && !r->fused && !r->scheme) {
        // the source and receivers run in the boundary kernel's last block
        return timed(1, [&] {
            return launch_boundary<T>(r->MB, r->idx64, r->bpos, r->Kb, r->matb, 0, r->nb, r->nb, un,
                                      ub_slot<T>(r, cur), (T *)r->gst, (T *)r->vst, (const T *)r->tab, (const T *)r->tab_host.data(), r->M,
                                      r->lambda, s, 0, 0, ctl_of<T>(r), r->ticket);
        });
    }
    return timed(2, [&] { return launch_src_rcv<T>(un, ub_slot<T>(r, cur), ctl_of<T>(r), s); });
}

// one double step of the two-step kernel (twostep.cu) from the state (pair,
// cur): A = u^{n-1}, B = u^n -> C = u^{n+1}, D = u^{n+2} in the other pair,
// placed so that the state after it is (pair^2, cur).  The u_b slots follow
// the steps (slot cur for step n+1, cur^1 for step n+2), as two single steps.
template <typename T> static cudaError_t enqueue_step2(rafd_room *r, int pair, int cur, cudaStream_t s, bool prof)
{
    const Grid &g = r->g;
    const int bA = pair + (cur ^ 1), bB = pair + cur, bC = (pair ^ 2) + (cur ^ 1), bD = (pair ^ 2) + cur;
    T *B = (T *)r->u[bB], *C = (T *)r->u[bC], *D = (T *)r->u[bD];
    // boundary update + (in its last block) source and receivers of one step;
    // without boundary nodes the source/receiver kernel alone
    auto bnd_src = [&](T *un, int slot) -> cudaError_t {
        if (r->nb == 0)
            return timed_launch(r, s, prof, 2, [&] { return launch_src_rcv<T>(un, ub_slot<T>(r, slot), ctl_of<T>(r), s); });
        return timed_launch(r, s, prof, 1, [&] {
            return launch_boundary<T>(r->MB, r->idx64, r->bpos, r->Kb, r->matb, 0, r->nb, r->nb, un,
                                      ub_slot<T>(r, slot), (T *)r->gst, (T *)r->vst, (const T *)r->tab, (const T *)r->tab_host.data(), r->M,
                                      r->lambda, s, 0, 0, ctl_of<T>(r), r->ticket);
        });
    };
    cudaError_t e = timed_launch(r, s, prof, 0, [&] { return launch_volume2<T>(r->tbplan, g, bB, bA, C, D, r->lambda, s); });
    if (e == cudaSuccess) e = bnd_src(C, cur);
    if (e == cudaSuccess && r->shell_bnd) {
        // the shell, the step-(n+2) boundary update and the source / receivers in one pass
        return timed_launch(r, s, prof, 3, [&] {
            return launch_shell_bnd<T>(r->tbplan, g, C, B, r->K, D, r->lambda, r->MB, r->matb, ub_slot<T>(r, cur ^ 1),
                                       (T *)r->gst, (T *)r->vst, r->nb, (const T *)r->tab, r->M, ctl_of<T>(r),
                                       r->ticket, s);
        });
    }
    if (e == cudaSuccess)
        e = timed_launch(r, s, prof, 3, [&] { return launch_shell<T>(r->tbplan, g, C, B, r->K, D, r->lambda, s); });
    if (e == cudaSuccess) e = bnd_src(D, cur ^ 1);
    return e;
}

// ---- slab step, edge planes first: phase 0 = the first and
// last owned plane (volume, their boundary nodes, the source if it lies there),
// then the halo exchange runs on comm_stream while phase 1 = the interior
// planes (volume, boundary nodes, source, receivers) runs on the main stream.
// mirror (halo push): byte offsets to the lower / upper neighbour's ghost plane
// for the phase-0 stores (null = no push)
template <typename T>
static cudaError_t enqueue_phase(rafd_room *r, int phase, cudaStream_t s, bool prof, const int64_t *mirror = nullptr)
{
    const Grid &g = r->g;
    const int lnz = g.lnz, cur = r->cur, pc = r->pair + r->cur;
    T *uc = (T *)r->u[pc];
    T *un = (T *)r->u[pc ^ 1];
    auto timed = [&](int kind, auto fn) -> cudaError_t { return timed_launch(r, s, prof, kind, fn); };
    const FusedArgs<T> fa = fused_args<T>(r);
    // mirrors of the first owned plane (to the lower neighbour) and the last (to the upper one)
    const int64_t m_lo = mirror ? mirror[0] : 0, m_hi = mirror ? mirror[1] : 0;
    const int64_t mf0 = m_lo, mf1 = lnz == 1 ? m_hi : 0;  // plane 0 (and the last, if it is the same)
    auto vol = [&](int zl, int zh, int64_t m0, int64_t m1) {
        FusedArgs<T> f = fa;
        f.mirror[0] = m0;
        f.mirror[1] = m1;
        return timed(0, [&] {
            return launch_volume<T>(g, uc, un, r->K, r->lambda, zl, zh, s, r->vplan, pc,
                                    (r->fused || r->scheme || m0 || m1) ? &f : nullptr);
        });
    };
    auto bnd = [&](int64_t lo, int64_t hi, int64_t m0, int64_t m1, int src_mode = 0) -> cudaError_t {
        if (hi <= lo || r->fused || r->scheme) return cudaSuccess;
        return timed(1, [&] {
            return launch_boundary<T>(r->MB, r->idx64, r->bpos, r->Kb, r->matb, lo, hi, r->nb, un,
                                      ub_slot<T>(r, cur), (T *)r->gst, (T *)r->vst, (const T *)r->tab, (const T *)r->tab_host.data(), r->M,
                                      r->lambda, s, m0, m1, src_mode ? ctl_of<T>(r) : nullptr, r->ticket,
                                      src_mode);
        });
    };
    const int zs = r->src_z >= 0 ? r->src_z - r->z0 : -1;
    const bool src_edge = zs == 0 || zs == lnz - 1;
    // the interior phase's source/receivers run in the interior boundary kernel's
    // last block when that kernel runs
    const bool bnd_src = !r->fused && !r->scheme && lnz > 2 && r->n_last_start > r->n_first_plane;
    cudaError_t e = cudaSuccess;
    if (phase == 0) {
        e = vol(0, 1, mf0, mf1);
        if (e == cudaSuccess && lnz > 1) e = vol(lnz - 1, lnz, m_hi, 0);
        if (e == cudaSuccess) e = bnd(0, std::min(r->n_first_plane, r->nb), mf0, mf1);
        if (e == cudaSuccess && lnz > 1) e = bnd(std::max(r->n_last_start, r->n_first_plane), r->nb, m_hi, 0);
        const int64_t ms0 = zs == 0 ? mf0 : m_hi, ms1 = zs == 0 ? mf1 : 0;
        if (e == cudaSuccess && src_edge)
            e = timed(2, [&] { return launch_src_rcv<T>(un, ub_slot<T>(r, cur), ctl_of<T>(r), s, 1, ms0, ms1); });
    } else {
        if (lnz > 2) e = vol(1, lnz - 1, 0, 0);
        if (e == cudaSuccess && lnz > 2) e = bnd(r->n_first_plane, r->n_last_start, 0, 0, bnd_src ? (src_edge ? 2 : 3) : 0);
        if (e == cudaSuccess && !bnd_src)
            e = timed(2, [&] { return launch_src_rcv<T>(un, ub_slot<T>(r, cur), ctl_of<T>(r), s, src_edge ? 2 : 3); });
    }
    return e;
}

static int kernels_per_phase(const rafd_room *r, int phase)
{
    const int lnz = r->g.lnz;
    const int nbk = (r->fused || r->scheme) ? 0 : 1;  // boundary launches exist only in the two-kernel form
    if (phase == 0) {
        const int zs = r->src_z >= 0 ? r->src_z - r->z0 : -1;
        return (lnz > 1 ? 2 : 1) + nbk * (r->n_first_plane > 0 ? 1 : 0) +
               nbk * (lnz > 1 && r->nb > std::max(r->n_last_start, r->n_first_plane) ? 1 : 0) +
               ((zs == 0 || zs == lnz - 1) ? 1 : 0);
    }
    // interior volume, then either the interior boundary kernel (which runs the
    // source/receivers in its last block) or k_src_rcv alone; the second
    // interior phase of a double step (ph 3) is one fused shell + boundary
    // launch when the slab has interior nodes
    if (phase == 3 && r->shell_bnd && lnz > 2 && r->n_last_start > r->n_first_plane) return 1;
    return (lnz > 2 ? 1 : 0) + 1;
}

// ---- slab double step under temporal blocking (twostep.cu), from the state
// (pair, cur): A = u^{n-1}, B = u^n -> C = u^{n+1}, D = u^{n+2} in the other
// pair.  The two-step kernel needs u^n one plane beyond the planes it
// advances, and u^{n+1} of the edge planes is final only after the
// neighbours' boundary nodes and source of step n+1 -- so a slab runs:
//   ph 0 (E1): u^{n+1} of the first / last owned plane with the single-step
//              kernel (B, A -> C), their boundary nodes (u_b slot cur), the
//              source if it lies there; then C's edge planes are exchanged
//   ph 1 (I1): the two-step kernel over the interior planes [1, lnz-1) (B, A
//              -> C, D; it recomputes u^{n+1} of the edge planes for itself,
//              unstored), their boundary nodes, the source, the receivers
//   ph 2 (E2): after the exchange, u^{n+2} of the edge planes (C, B -> D),
//              their boundary nodes (slot cur^1), the source; D's edge planes
//              are exchanged
//   ph 3 (I2): the shell of the interior planes (C, B -> D), their boundary
//              nodes, the source, the receivers.
// Every value is the single-step expression on the same operands: bitwise
// the undivided room.  One plane per neighbour per step is exchanged, as with
// single steps; the first exchange hides behind the two-step kernel.
template <typename T>
static cudaError_t enqueue_tb_phase(rafd_room *r, int ph, cudaStream_t s, bool prof, const int64_t *mirror = nullptr)
{
    const Grid &g = r->g;
    const int lnz = g.lnz, pair = r->pair, cur = r->cur;
    const int bA = pair + (cur ^ 1), bB = pair + cur, bC = (pair ^ 2) + (cur ^ 1), bD = (pair ^ 2) + cur;
    const bool second = ph >= 2;
    const int bu = second ? bC : bB, bp = second ? bB : bA, bo = second ? bD : bC;
    T *out = (T *)r->u[bo];
    T *ub = ub_slot<T>(r, second ? cur ^ 1 : cur);
    auto timed = [&](int kind, auto fn) -> cudaError_t { return timed_launch(r, s, prof, kind, fn); };
    const int64_t m_lo = mirror ? mirror[0] : 0, m_hi = mirror ? mirror[1] : 0;
    const int64_t mf0 = m_lo, mf1 = lnz == 1 ? m_hi : 0;
    auto vol = [&](int zl, int zh, int64_t m0, int64_t m1) {
        FusedArgs<T> f = fused_args<T>(r);
        f.mirror[0] = m0;
        f.mirror[1] = m1;
        return timed(0, [&] {
            return launch_volume<T>(g, (const T *)r->u[bu], out, r->K, r->lambda, zl, zh, s, r->vplan, bu,
                                    (m0 || m1) ? &f : nullptr, bp);
        });
    };
    auto bnd = [&](int64_t lo, int64_t hi, int64_t m0, int64_t m1, int src_mode = 0) -> cudaError_t {
        if (hi <= lo) return cudaSuccess;
        return timed(1, [&] {
            return launch_boundary<T>(r->MB, r->idx64, r->bpos, r->Kb, r->matb, lo, hi, r->nb, out, ub, (T *)r->gst,
                                      (T *)r->vst, (const T *)r->tab, (const T *)r->tab_host.data(), r->M, r->lambda, s, m0, m1,
                                      src_mode ? ctl_of<T>(r) : nullptr, r->ticket, src_mode);
        });
    };
    const bool bnd_src = lnz > 2 && r->n_last_start > r->n_first_plane;  // see enqueue_phase
    const int zs = r->src_z >= 0 ? r->src_z - r->z0 : -1;
    const bool src_edge = zs == 0 || zs == lnz - 1;
    cudaError_t e = cudaSuccess;
    if (ph == 0 || ph == 2) {
        e = vol(0, 1, mf0, mf1);
        if (e == cudaSuccess && lnz > 1) e = vol(lnz - 1, lnz, m_hi, 0);
        if (e == cudaSuccess) e = bnd(0, std::min(r->n_first_plane, r->nb), mf0, mf1);
        if (e == cudaSuccess && lnz > 1) e = bnd(std::max(r->n_last_start, r->n_first_plane), r->nb, m_hi, 0);
        const int64_t ms0 = zs == 0 ? mf0 : m_hi, ms1 = zs == 0 ? mf1 : 0;
        if (e == cudaSuccess && src_edge)
            e = timed(2, [&] { return launch_src_rcv<T>(out, ub, ctl_of<T>(r), s, 1, ms0, ms1); });
    } else {
        if (lnz > 2 && ph == 3 && r->shell_bnd && bnd_src) {
            // the interior shell, its boundary nodes and the source / receivers in one pass
            return timed(3, [&] {
                return launch_shell_bnd<T>(r->tbplan, g, (const T *)r->u[bC], (const T *)r->u[bB], r->K,
                                           (T *)r->u[bD], r->lambda, r->MB, r->matb, ub, (T *)r->gst, (T *)r->vst,
                                           r->nb, (const T *)r->tab, r->M, ctl_of<T>(r), r->ticket, s, true,
                                           src_edge ? 2 : 3);
            });
        }
        if (lnz > 2) {
            if (ph == 1)
                e = timed(0, [&] {
                    return launch_volume2<T>(r->tbplan, g, bB, bA, (T *)r->u[bC], (T *)r->u[bD], r->lambda, s, 1,
                                             lnz - 1);
                });
            else
                e = timed(3, [&] {
                    return launch_shell<T>(r->tbplan, g, (const T *)r->u[bC], (const T *)r->u[bB], r->K,
                                           (T *)r->u[bD], r->lambda, s, true);
                });
        }
        if (e == cudaSuccess && lnz > 2)
            e = bnd(r->n_first_plane, r->n_last_start, 0, 0, bnd_src ? (src_edge ? 2 : 3) : 0);
        if (e == cudaSuccess && !bnd_src)
            e = timed(2, [&] { return launch_src_rcv<T>(out, ub, ctl_of<T>(r), s, src_edge ? 2 : 3); });
    }
    return e;
}

// the slab phase `ph` of a single step (0, 1) or of a double step (0..3), and
// the field buffer whose edge planes the exchange after phase ph (even) sends
static cudaError_t slab_phase(rafd_room *r, bool two, int ph, cudaStream_t s, bool prof, const int64_t *mirror = nullptr)
{
    if (two)
        return r->prec == 32 ? enqueue_tb_phase<float>(r, ph, s, prof, mirror)
                             : enqueue_tb_phase<double>(r, ph, s, prof, mirror);
    return r->prec == 32 ? enqueue_phase<float>(r, ph, s, prof, mirror) : enqueue_phase<double>(r, ph, s, prof, mirror);
}
static int exchange_buf(const rafd_room *r, bool two, int ph)
{
    if (!two) return r->pair + (r->cur ^ 1);
    return ph < 2 ? (r->pair ^ 2) + (r->cur ^ 1) : (r->pair ^ 2) + r->cur;
}

// One step (two = false) or double step (two = true) of a z slab with its
// halo transport; n = steps taken so far (the IPC signal words count steps:
// exactly one exchange per step in both modes).
//  * NCCL: after the edge phase, ncclSend/ncclRecv of the edge planes on
//    comm_stream, overlapped with the interior phase; the next edge phase
//    waits for it.
//  * IPC pull: the edge phase publishes word 0 = m+1; comm_stream waits for
//    the neighbours' word 0, copies their edge planes into my ghost planes
//    (peer copies) and publishes word 1 = m+1; an edge phase first waits for
//    the neighbours' word 1 >= m (WAR: they finished copying out of my
//    buffers).
//  * IPC push: the edge-phase kernels also store their
//    planes into the neighbours' ghost planes over peer memory, then one
//    fenced signal word 0 = m+1; the edge phase of step m first waits for the
//    neighbours' word 0 >= m, which orders both the ghost reads (RAW) and the
//    next pushes (WAR: a ghost plane is last read in the edge phase -- or the
//    two-step kernel right after it -- of an earlier step).
static cudaError_t slab_step(rafd_room *r, bool two, bool prof, int64_t n)
{
    cudaError_t e = cudaSuccess;
    const size_t pb = (size_t)r->g.plane * r->s;
    const int lnz = r->g.lnz;
    for (int h = 0; h < (two ? 2 : 1); h++) {
        const int64_t m = n + h;
        const int pe = two ? 2 * h : 0, pi = pe + 1;
        const int xb = exchange_buf(r, two, pe);
        if (r->ipc && r->push) {
            if (m > 0 && (e = ipc_wait_peers(r->ipc, 0, m, r->stream)) != cudaSuccess) return e;
            int64_t mr[2];
            ipc_mirror_deltas(r->ipc, xb, r->u[xb], pb, lnz, &mr[0], &mr[1]);
            if ((e = slab_phase(r, two, pe, r->stream, prof, mr)) != cudaSuccess) return e;
            if ((e = ipc_signal(r->ipc_sig + 0, m + 1, r->stream)) != cudaSuccess) return e;  // with a memory fence
            if ((e = slab_phase(r, two, pi, r->stream, prof)) != cudaSuccess) return e;
            continue;
        }
        if (r->ipc && m > 0 && (e = ipc_wait_peers(r->ipc, 1, m, r->stream)) != cudaSuccess) return e;
        if ((e = slab_phase(r, two, pe, r->stream, prof)) != cudaSuccess) return e;
        if (r->ipc && (e = ipc_signal(r->ipc_sig + 0, m + 1, r->stream)) != cudaSuccess) return e;
        if ((e = cudaEventRecord(r->ev_edge, r->stream)) != cudaSuccess) return e;
        if ((e = cudaStreamWaitEvent(r->comm_stream, r->ev_edge, 0)) != cudaSuccess) return e;
        if (r->ipc) {
            if ((e = ipc_wait_peers(r->ipc, 0, m + 1, r->comm_stream)) != cudaSuccess) return e;
            if ((e = ipc_pull(r->ipc, xb, r->u[xb], pb, lnz, r->comm_stream)) != cudaSuccess) return e;
            if ((e = ipc_signal(r->ipc_sig + 1, m + 1, r->comm_stream)) != cudaSuccess) return e;
        } else {
            if ((e = halo_exchange(r->halo, r->u[xb], pb, lnz, r->comm_stream)) != cudaSuccess) return e;
        }
        if ((e = cudaEventRecord(r->ev_halo, r->comm_stream)) != cudaSuccess) return e;
        if ((e = slab_phase(r, two, pi, r->stream, prof)) != cudaSuccess) return e;
        if ((e = cudaStreamWaitEvent(r->stream, r->ev_halo, 0)) != cudaSuccess) return e;  // ghost planes ready
    }
    return e;
}

// (whole room: the boundary kernel runs the source/receivers in its last block;
// fused / single-kernel schemes and rooms without boundary nodes launch k_src_rcv)
static int kernels_per_step(const rafd_room *) { return 2; }
// k_volume2, the step-(n+1) boundary kernel, and the shell + step-(n+2)
// boundary (fused: one kernel; else two)
static int kernels_per_double_step(const rafd_room *r) { return r->shell_bnd ? 3 : 4; }

// a graph of G steps from the state (pair, cur) (index pair + cur); it ends in
// the same state (G single steps flip cur an even number of times, G/2 double
// steps flip pair an even number of times)
template <typename T> static int build_graph(rafd_room *r, int pair, int cur)
{
    cudaGraph_t gr;
    CK(cudaStreamBeginCapture(r->cap_stream, cudaStreamCaptureModeThreadLocal));
    cudaError_t e = cudaSuccess;
    if (r->tb == 2) {
        for (int k = 0; k < rafd_room::G / 2 && e == cudaSuccess; k++)
            e = enqueue_step2<T>(r, pair ^ (2 * (k & 1)), cur, r->cap_stream, false);
    } else {
        for (int k = 0; k < rafd_room::G && e == cudaSuccess; k++)
            e = enqueue_step<T>(r, pair, cur ^ (k & 1), r->cap_stream, false);
    }
    cudaError_t e2 = cudaStreamEndCapture(r->cap_stream, &gr);
    if (e != cudaSuccess) return set_err(RAFD_E_CUDA, "capture: %s", cudaGetErrorString(e));
    CK(e2);
    CK(cudaGraphInstantiate(&r->graph[pair + cur], gr, 0));
    cudaGraphDestroy(gr);
    return RAFD_OK;
}

template <typename T> static int step_t(rafd_room *r, int64_t nsteps)
{
    int rc = ensure_rec<T>(r, nsteps);
    if (rc) return rc;
    const int kps = kernels_per_step(r);
    int64_t done = 0;
    const bool use_graph = !r->profiling && !r->halo && !r->ipc && nsteps >= rafd_room::G;
    const int gi = r->pair + r->cur;
    while (use_graph && nsteps - done >= rafd_room::G) {
        if (!r->graph[gi] && (rc = build_graph<T>(r, r->pair, r->cur))) return rc;
        CK(cudaGraphLaunch(r->graph[gi], r->stream));
        done += rafd_room::G;  // G is even: state unchanged
        r->launches += r->tb == 2 ? (int64_t)kernels_per_double_step(r) * (rafd_room::G / 2) : (int64_t)kps * rafd_room::G;
    }
    // temporal blocking: double steps, an odd last step runs single
    const bool slab = r->halo || r->ipc;
    auto slab_err = [&](cudaError_t e) {
        if (e == cudaErrorUnknown) return set_err(r->halo ? RAFD_E_NCCL : RAFD_E_CUDA, "%s", halo_last_error());
        return set_err(RAFD_E_CUDA, "step: %s", cudaGetErrorString(e));
    };
    const int64_t kslab = slab ? kernels_per_phase(r, 0) + kernels_per_phase(r, 1) : 0;
    const int64_t kslab2 = slab ? 2 * kernels_per_phase(r, 0) + kernels_per_phase(r, 1) + kernels_per_phase(r, 3) : 0;
    while (r->tb == 2 && nsteps - done >= 2) {
        cudaError_t e = slab ? slab_step(r, true, r->profiling, r->steps + done)
                             : enqueue_step2<T>(r, r->pair, r->cur, r->stream, r->profiling);
        if (e != cudaSuccess) return slab ? slab_err(e) : set_err(RAFD_E_CUDA, "step: %s", cudaGetErrorString(e));
        r->launches += slab ? kslab2 : kernels_per_double_step(r);
        r->pair ^= 2;
        done += 2;
    }
    for (; done < nsteps; done++) {
        if (slab) {
            cudaError_t e = slab_step(r, false, r->profiling, r->steps + done);
            if (e != cudaSuccess) return slab_err(e);
            r->launches += kslab;
        } else {
            cudaError_t e = enqueue_step<T>(r, r->pair, r->cur, r->stream, r->profiling);
            if (e != cudaSuccess) return set_err(RAFD_E_CUDA, "step: %s", cudaGetErrorString(e));
            r->launches += kps;
        }
        r->cur ^= 1;
    }
    r->steps += nsteps;
    if (r->nrcv > 0) r->rec_count += nsteps;
    return RAFD_OK;
}

extern "C" int rafd_step(rafd_room *r, int64_t nsteps)
{
    if (!r || nsteps < 0) return set_err(RAFD_E_INVAL, "bad step arguments");
    if (r->local_slab && !r->ipc)
        return set_err(RAFD_E_STATE, "a slab created without nccl_id is stepped with rafd_step_group or after rafd_ipc_connect");
    if (nsteps == 0) return RAFD_OK;
    CK(cudaSetDevice(r->device));
    return r->prec == 32 ? step_t<float>(r, nsteps) : step_t<double>(r, nsteps);
}

// Slabs of one room held by this process (one per device, or several on one
// device): every step, each slab runs its kernels on its own stream, then pulls
// its two ghost planes from its neighbours' current u buffers (cudaMemcpyAsync,
// peer copy across devices), ordered by events; a slab's next step waits for
// its neighbours' copies out of its buffer.  Results are identical to one room.
template <typename T> static int step_group_t(rafd_room **rs, int n, int64_t nsteps)
{
    for (int k = 0; k < n; k++) {
        int rc = ensure_rec<T>(rs[k], nsteps);
        if (rc) return rc;
    }
    const bool tb2 = rs[0]->tb == 2;  // temporal blocking: double steps (enqueue_tb_phase), an odd last one single
    for (int64_t done = 0; done < nsteps;) {
        const bool two = tb2 && nsteps - done >= 2;
        for (int h = 0; h < (two ? 2 : 1); h++) {
            const int pe = two ? 2 * h : 0;
            // edge phase of every slab, after the neighbours finished copying
            // out of its buffers (their previous pulls)
            for (int k = 0; k < n; k++) {
                rafd_room *r = rs[k];
                CK(cudaSetDevice(r->device));
                if (k > 0) CK(cudaStreamWaitEvent(r->stream, rs[k - 1]->ev_halo, 0));
                if (k < n - 1) CK(cudaStreamWaitEvent(r->stream, rs[k + 1]->ev_halo, 0));
                cudaError_t e = slab_phase(r, two, pe, r->stream, r->profiling);
                if (e != cudaSuccess) return set_err(RAFD_E_CUDA, "step: %s", cudaGetErrorString(e));
                CK(cudaEventRecord(r->ev_edge, r->stream));
                r->launches += kernels_per_phase(r, 0);
            }
            // halo: each slab pulls its ghost planes on its comm stream
            for (int k = 0; k < n; k++) {
                rafd_room *r = rs[k];
                CK(cudaSetDevice(r->device));
                const size_t pb = (size_t)r->g.plane * sizeof(T);
                char *mine = (char *)r->u[exchange_buf(r, two, pe)];
                CK(cudaStreamWaitEvent(r->comm_stream, r->ev_edge, 0));
                if (k > 0) {
                    rafd_room *q = rs[k - 1];
                    CK(cudaStreamWaitEvent(r->comm_stream, q->ev_edge, 0));
                    const char *src = (const char *)q->u[exchange_buf(q, two, pe)] + (size_t)q->g.lnz * pb;
                    CK(cudaMemcpyPeerAsync(mine, r->device, src, q->device, pb, r->comm_stream));
                }
                if (k < n - 1) {
                    rafd_room *q = rs[k + 1];
                    CK(cudaStreamWaitEvent(r->comm_stream, q->ev_edge, 0));
                    const char *src = (const char *)q->u[exchange_buf(q, two, pe)] + pb;
                    CK(cudaMemcpyPeerAsync(mine + (size_t)(r->g.lnz + 1) * pb, r->device, src, q->device, pb,
                                           r->comm_stream));
                }
                CK(cudaEventRecord(r->ev_halo, r->comm_stream));
            }
            // interior phase overlapped with the copies
            for (int k = 0; k < n; k++) {
                rafd_room *r = rs[k];
                CK(cudaSetDevice(r->device));
                cudaError_t e = slab_phase(r, two, pe + 1, r->stream, r->profiling);
                if (e != cudaSuccess) return set_err(RAFD_E_CUDA, "step: %s", cudaGetErrorString(e));
                CK(cudaStreamWaitEvent(r->stream, r->ev_halo, 0));
                r->launches += kernels_per_phase(r, two ? pe + 1 : 1);
            }
        }
        for (int k = 0; k < n; k++) {
            if (two) rs[k]->pair ^= 2;
            else rs[k]->cur ^= 1;
        }
        done += two ? 2 : 1;
    }
    for (int k = 0; k < n; k++) {
        rs[k]->steps += nsteps;
        if (rs[k]->nrcv > 0) rs[k]->rec_count += nsteps;
    }
    return RAFD_OK;
}

extern "C" int rafd_step_group(rafd_room **rooms, int32_t n, int64_t nsteps)
{
    if (!rooms || n < 1 || nsteps < 0) return set_err(RAFD_E_INVAL, "bad group arguments");
    for (int k = 0; k < n; k++) {
        rafd_room *r = rooms[k];
        if (!r) return set_err(RAFD_E_INVAL, "null room in group");
        if (n == 1 ? r->nranks != 1 : (!r->local_slab || r->nranks != n || r->rank != k))
            return set_err(RAFD_E_STATE, "group member %d is not local slab %d of %d", k, k, n);
        if (r->prec != rooms[0]->prec || r->nx != rooms[0]->nx || r->ny != rooms[0]->ny || r->nz != rooms[0]->nz)
            return set_err(RAFD_E_STATE, "group members are not slabs of one room");
        if (r->tb != rooms[0]->tb) return set_err(RAFD_E_STATE, "group members differ in steps_per_sweep");
        if (k > 0 && rooms[k - 1]->z1 != r->z0) return set_err(RAFD_E_STATE, "slabs are not contiguous");
    }
    if (nsteps == 0) return RAFD_OK;
    if (n == 1) return rafd_step(rooms[0], nsteps);
    // peer access between distinct devices (best effort; cudaMemcpyPeerAsync works without it)
    for (int k = 0; k + 1 < n; k++) {
        const int a = rooms[k]->device, b = rooms[k + 1]->device;
        if (a != b) {
            int can = 0;
            cudaDeviceCanAccessPeer(&can, a, b);
            if (can) {
                cudaSetDevice(a);
                cudaDeviceEnablePeerAccess(b, 0);
                cudaSetDevice(b);
                cudaDeviceEnablePeerAccess(a, 0);
                cudaGetLastError();
            }
        }
    }
    return rooms[0]->prec == 32 ? step_group_t<float>(rooms, n, nsteps) : step_group_t<double>(rooms, n, nsteps);
}

extern "C" int rafd_ipc_handle(rafd_room *r, uint8_t *blob)
{
    if (!r || !blob) return set_err(RAFD_E_INVAL, "bad arguments");
    if (!r->local_slab || !r->ipc_sig) return set_err(RAFD_E_STATE, "IPC handles exist for slabs created without nccl_id");
    CK(cudaSetDevice(r->device));
    int rc = ipc_make_blob(r->u, r->ipc_sig, r->device, r->g.lnz, (uint32_t)r->g.pitch, blob);
    if (rc) return set_err(rc, "%s", halo_last_error());
    return RAFD_OK;
}

extern "C" int rafd_ipc_connect(rafd_room *r, const uint8_t *lower, const uint8_t *upper)
{
    if (!r) return set_err(RAFD_E_INVAL, "null room");
    if (!r->local_slab || r->ipc) return set_err(RAFD_E_STATE, "rafd_ipc_connect: not an unconnected slab");
    if ((r->rank > 0) != (lower != nullptr) || (r->rank < r->nranks - 1) != (upper != nullptr))
        return set_err(RAFD_E_INVAL, "rank %d of %d needs %s lower and %s upper neighbour", r->rank, r->nranks,
                       r->rank > 0 ? "a" : "no", r->rank < r->nranks - 1 ? "an" : "no");
    CK(cudaSetDevice(r->device));
    CK(cudaStreamSynchronize(r->stream));
    int rc = ipc_open(&r->ipc, lower, upper, (uint32_t)r->g.pitch);
    if (rc) return set_err(rc, "%s", halo_last_error());
    return RAFD_OK;
}

extern "C" int rafd_set_halo_push(rafd_room *r, int32_t on)
{
    if (!r) return set_err(RAFD_E_INVAL, "null room");
    if (!on) {
        r->push = false;
        return RAFD_OK;
    }
    if (!r->ipc) return set_err(RAFD_E_STATE, "halo push needs an IPC-connected slab (rafd_ipc_connect)");
    if (r->fused || r->scheme || !r->vplan)
        return set_err(RAFD_E_STATE, "halo push runs with the two-kernel scheme and the TMA volume kernel");
    if (r->steps != 0) return set_err(RAFD_E_STATE, "choose the halo transport before the first step");
    r->push = true;
    return RAFD_OK;
}

extern "C" int rafd_synchronize(rafd_room *r)
{
    if (!r) return set_err(RAFD_E_INVAL, "null room");
    CK(cudaSetDevice(r->device));
    CK(cudaStreamSynchronize(r->stream));
    return RAFD_OK;
}

// ------------------------------------------------------------------ reads
// One stream-ordered D2H of the unread rows into a pinned staging buffer, a
// device-side reset of the row counter, one synchronisation (the host already
// knows how many rows the device wrote).
template <typename T> static int read_receivers_t(rafd_room *r, double *out, int64_t cap, int64_t *nw)
{
    const int64_t n = r->rec_count;
    if (r->nrcv > 0 && (cap < n || !out)) return set_err(RAFD_E_INVAL, "cap (%lld) < unread samples (%lld)", (long long)cap, (long long)n);
    const size_t bytes = (size_t)n * r->nrcv * sizeof(T);
    if (r->nrcv > 0 && n > 0) {
        if (r->rec_host_bytes < bytes) {
            if (r->rec_host) cudaFreeHost(r->rec_host);
            r->rec_host = nullptr;
            r->rec_host_bytes = 0;
            CK(cudaMallocHost(&r->rec_host, bytes));
            r->rec_host_bytes = bytes;
        }
        CK(cudaMemcpyAsync(r->rec_host, r->rec, bytes, cudaMemcpyDeviceToHost, r->stream));
    }
    CK(cudaMemsetAsync(&ctl_of<T>(r)->rec_count, 0, sizeof(int64_t), r->stream));
    CK(cudaStreamSynchronize(r->stream));
    if (r->nrcv > 0 && n > 0) {
        const T *h = (const T *)r->rec_host;
        for (int j = 0; j < r->nrcv; j++)
            for (int64_t k = 0; k < n; k++) out[j * cap + k] = (double)h[(size_t)k * r->nrcv + j];
    }
    *nw = r->nrcv > 0 ? n : 0;
    r->rec_count = 0;
    return RAFD_OK;
}

extern "C" int rafd_read_receivers(rafd_room *r, double *out, int64_t cap, int64_t *n_written)
{
    if (!r || !n_written) return set_err(RAFD_E_INVAL, "bad arguments");
    CK(cudaSetDevice(r->device));
    return r->prec == 32 ? read_receivers_t<float>(r, out, cap, n_written)
                         : read_receivers_t<double>(r, out, cap, n_written);
}

template <typename T> static int field_out_t(rafd_room *r, const T *src, void *dst)
{
    const bool dev = is_device_ptr(dst);
    const size_t pb = (size_t)r->nx * r->ny * sizeof(T);
    const int lnz = r->g.lnz;
    if (dev) {
        CK(launch_field_out<T>(r->g, src, 1, lnz, (T *)dst, r->stream));
        CK(cudaStreamSynchronize(r->stream));
        return RAFD_OK;
    }
    void *st = nullptr;
    CK(cudaMalloc(&st, kStagingBytes));
    const int per = (int)std::max<size_t>(1, kStagingBytes / pb);
    for (int z = 0; z < lnz; z += per) {
        const int n = std::min(per, lnz - z);
        cudaError_t e = launch_field_out<T>(r->g, src, 1 + z, n, (T *)st, r->stream);
        if (e == cudaSuccess) e = cudaMemcpyAsync((char *)dst + (size_t)z * pb, st, (size_t)n * pb, cudaMemcpyDeviceToHost, r->stream);
        if (e == cudaSuccess) e = cudaStreamSynchronize(r->stream);
        if (e != cudaSuccess) {
            cudaFree(st);
            return set_err(RAFD_E_CUDA, "read_field: %s", cudaGetErrorString(e));
        }
    }
    cudaFree(st);
    return RAFD_OK;
}

extern "C" int rafd_read_field(rafd_room *r, void *u_curr, void *u_prev)
{
    if (!r) return set_err(RAFD_E_INVAL, "null room");
    CK(cudaSetDevice(r->device));
    int rc = RAFD_OK;
    const int bc = r->pair + r->cur, bp = r->pair + (r->cur ^ 1);
    if (u_curr) rc = r->prec == 32 ? field_out_t<float>(r, (const float *)r->u[bc], u_curr)
                                   : field_out_t<double>(r, (const double *)r->u[bc], u_curr);
    if (!rc && u_prev) rc = r->prec == 32 ? field_out_t<float>(r, (const float *)r->u[bp], u_prev)
                                          : field_out_t<double>(r, (const double *)r->u[bp], u_prev);
    return rc;
}

extern "C" int rafd_read_branch_state(rafd_room *r, void *v, void *g)
{
    if (!r) return set_err(RAFD_E_INVAL, "null room");
    CK(cudaSetDevice(r->device));
    CK(cudaStreamSynchronize(r->stream));
    const size_t n = (size_t)r->nb * r->MB * r->s;
    if (n == 0) return RAFD_OK;
    if (v) CK(cudaMemcpy(v, r->vst, n, cudaMemcpyDefault));
    if (g) CK(cudaMemcpy(g, r->gst, n, cudaMemcpyDefault));
    return RAFD_OK;
}

extern "C" int rafd_get_classification(rafd_room *r, uint8_t *K, int64_t *bidx, uint8_t *Kb, uint8_t *matb)
{
    if (!r) return set_err(RAFD_E_INVAL, "null room");
    CK(cudaSetDevice(r->device));
    CK(cudaStreamSynchronize(r->stream));
    if (K) {
        const size_t pb = (size_t)r->nx * r->ny;
        uint8_t *st = nullptr;
        CK(cudaMalloc((void **)&st, pb * r->g.lnz + 16));
        CK(launch_field_out<uint8_t>(r->g, r->K, 1, r->g.lnz, st, r->stream));
        CK(cudaMemcpyAsync(K, st, pb * r->g.lnz, cudaMemcpyDefault, r->stream));
        CK(cudaStreamSynchronize(r->stream));
        cudaFree(st);
    }
    if (r->nb > 0) {
        if (bidx) CK(cudaMemcpy(bidx, r->bidx, (size_t)r->nb * 8, cudaMemcpyDefault));
        if (Kb) CK(cudaMemcpy(Kb, r->Kb, (size_t)r->nb, cudaMemcpyDefault));
        if (matb) CK(cudaMemcpy(matb, r->matb, (size_t)r->nb, cudaMemcpyDefault));
    }
    return RAFD_OK;
}

// ------------------------------------------------------------------ state in
template <typename T> static int field_in_t(rafd_room *r, const void *src, T *dst)
{
    // planes [z0-1, z1] of the room (ghost planes included when they exist)
    const bool dev = is_device_ptr(src);
    const size_t pb = (size_t)r->nx * r->ny * sizeof(T);
    const int zlo = std::max(0, r->z0 - 1), zhi = std::min(r->nz, r->z1 + 1);
    void *st = nullptr;
    if (!dev) CK(cudaMalloc(&st, kStagingBytes));
    int rc = for_plane_chunks(r, src, 0, dev, pb, zlo, zhi - zlo, st, kStagingBytes,
                              [&](const void *chunk, int zg, int n) -> int {
                                  CK(launch_field_in<T>(r->g, (const T *)chunk, zg - r->z0 + 1, n, r->K, dst, r->stream));
                                  return RAFD_OK;
                              });
    cudaStreamSynchronize(r->stream);
    if (st) cudaFree(st);
    return rc;
}

template <typename T> static int set_step_t(rafd_room *r, int64_t n)
{
    Ctl<T> c;
    int rc = pull_ctl<T>(r, c);
    if (rc) return rc;
    c.n = n;
    rc = push_ctl<T>(r, c);
    if (!rc) r->steps = n;
    return rc;
}

extern "C" int rafd_set_step(rafd_room *r, int64_t n)
{
    if (!r || n < 0) return set_err(RAFD_E_INVAL, "bad arguments");
    if (r->ipc) return set_err(RAFD_E_STATE, "the step counter of a connected IPC slab orders its signals");
    CK(cudaSetDevice(r->device));
    return r->prec == 32 ? set_step_t<float>(r, n) : set_step_t<double>(r, n);
}

// u_b slot `slot` <- field buffer u[buf] at the boundary nodes
static int gather_ub_slot(rafd_room *r, int buf, int slot)
{
    if (r->nb == 0) return RAFD_OK;
    if (r->prec == 32)
        CK(launch_gather_ub<float>(r->bpos, r->idx64, r->nb, (const float *)r->u[buf], (float *)r->ub + (int64_t)slot * r->nb, r->stream));
    else
        CK(launch_gather_ub<double>(r->bpos, r->idx64, r->nb, (const double *)r->u[buf], (double *)r->ub + (int64_t)slot * r->nb, r->stream));
    return RAFD_OK;
}

extern "C" int rafd_set_state(rafd_room *r, const void *u_prev, const void *u_curr, const void *v, const void *g)
{
    if (!r) return set_err(RAFD_E_INVAL, "null room");
    CK(cudaSetDevice(r->device));
    CK(cudaStreamSynchronize(r->stream));
    // device inputs may still be in flight on the caller's streams (see rafd_create)
    for (const void *p : {u_prev, u_curr, v, g})
        if (p && is_device_ptr(p)) {
            CK(cudaDeviceSynchronize());
            break;
        }
    int rc = RAFD_OK;
    const int bc = r->pair + r->cur, bp = r->pair + (r->cur ^ 1);
    if (u_prev) {
        rc = r->prec == 32 ? field_in_t<float>(r, u_prev, (float *)r->u[bp])
                           : field_in_t<double>(r, u_prev, (double *)r->u[bp]);
        if (rc) return rc;
        // u_b slot cur = u^{n-1} at the boundary nodes (reading R8)
        rc = gather_ub_slot(r, bp, r->cur);
        if (rc) return rc;
    }
    if (u_curr) {
        rc = r->prec == 32 ? field_in_t<float>(r, u_curr, (float *)r->u[bc])
                           : field_in_t<double>(r, u_curr, (double *)r->u[bc]);
        if (rc) return rc;
        rc = gather_ub_slot(r, bc, r->cur ^ 1);  // slot cur^1 = u^n (read by the next step)
        if (rc) return rc;
    }
    const size_t n = (size_t)r->nb * r->MB * r->s;
    if (n) {
        if (v) CK(cudaMemcpy(r->vst, v, n, cudaMemcpyDefault));
        if (g) CK(cudaMemcpy(r->gst, g, n, cudaMemcpyDefault));
    }
    CK(cudaStreamSynchronize(r->stream));
    return RAFD_OK;
}

// ------------------------------------------------------------------ info / energy / profiling
static void bytes_per_step(const rafd_room *r, int64_t *vol, int64_t *bnd)
{
    // B_step = N_mask*1 + N_in*3s + Nb*(6 + 3s + 4s*MB)
    const int64_t s = (int64_t)r->s;
    *vol = (int64_t)r->g.lnz * r->nx * r->ny + r->n_inside * 3 * s;
    *bnd = r->nb * (6 + 3 * s + 4 * s * r->MB);
}

extern "C" int rafd_get_info(rafd_room *r, rafd_info *info)
{
    if (!r || !info) return set_err(RAFD_E_INVAL, "bad arguments");
    memset(info, 0, sizeof *info);
    info->n_mask = (int64_t)r->g.lnz * r->nx * r->ny;
    info->n_inside = r->n_inside;
    info->n_boundary = r->nb;
    for (int k = 0; k < 7; k++) info->k_hist[k] = r->k_hist[k];
    info->isolated = r->isolated;
    info->steps = r->steps;
    bytes_per_step(r, &info->volume_bytes, &info->boundary_bytes);
    info->bytes_per_step = info->volume_bytes + info->boundary_bytes;
    info->device_bytes = r->device_bytes;
    info->precision = r->prec;
    info->n_materials = r->M;
    info->n_branches = r->MB;
    info->z_begin = r->z0;
    info->z_end = r->z1;
    info->pitch = (int32_t)r->g.pitch;
    info->fused = r->fused ? 1 : 0;
    info->scheme = r->scheme;
    info->steps_per_sweep = r->tb;
    info->n_shell = r->n_shell;
    return RAFD_OK;
}

extern "C" int rafd_energy(rafd_room *r, double *H)
{
    if (!r || !H) return set_err(RAFD_E_INVAL, "bad arguments");
    CK(cudaSetDevice(r->device));
    double *acc = nullptr;
    CK(cudaMalloc((void **)&acc, 3 * sizeof(double)));
    CK(cudaMemsetAsync(acc, 0, 3 * sizeof(double), r->stream));
    const void *un1 = r->u[r->pair + r->cur], *un = r->u[r->pair + (r->cur ^ 1)];
    cudaError_t e;
    if (r->prec == 32) {
        e = launch_energy<float>(r->g, (const float *)un1, (const float *)un, r->K, acc, r->stream);
        if (e == cudaSuccess) e = launch_energy_bnd<float>(r->Kb, r->matb, r->nb, r->MB, (const float *)r->vst, (const float *)r->gst, r->DF, r->M, r->lambda, acc, r->stream);
    } else {
        e = launch_energy<double>(r->g, (const double *)un1, (const double *)un, r->K, acc, r->stream);
        if (e == cudaSuccess) e = launch_energy_bnd<double>(r->Kb, r->matb, r->nb, r->MB, (const double *)r->vst, (const double *)r->gst, r->DF, r->M, r->lambda, acc, r->stream);
    }
    double h[3] = {0, 0, 0};
    if (e == cudaSuccess) e = cudaMemcpyAsync(h, acc, sizeof h, cudaMemcpyDeviceToHost, r->stream);
    if (e == cudaSuccess) e = cudaStreamSynchronize(r->stream);
    cudaFree(acc);
    if (e != cudaSuccess) return set_err(RAFD_E_CUDA, "energy: %s", cudaGetErrorString(e));
    *H = h[0] + r->lambda * r->lambda * h[1] + h[2];
    return RAFD_OK;
}

static void resolve_events(rafd_room *r)
{
    if (r->evs.empty()) return;
    cudaStreamSynchronize(r->stream);
    for (auto &e : r->evs) {
        float ms = 0;
        cudaEventElapsedTime(&ms, e.a, e.b);
        if (e.kind == 0) {
            r->kt.volume_ms += ms;
            r->kt.volume_n++;
        } else if (e.kind == 1) {
            r->kt.boundary_ms += ms;
            r->kt.boundary_n++;
        } else if (e.kind == 3) {
            r->kt.shell_ms += ms;
            r->kt.shell_n++;
        } else {
            r->kt.other_ms += ms;
            r->kt.other_n++;
        }
        r->ev_pool.push_back(e.a);
        r->ev_pool.push_back(e.b);
    }
    r->evs.clear();
}

extern "C" int rafd_set_profiling(rafd_room *r, int on)
{
    if (!r) return set_err(RAFD_E_INVAL, "null room");
    CK(cudaSetDevice(r->device));
    resolve_events(r);
    r->kt = KernelTimes();
    r->profiling = on != 0;
    return RAFD_OK;
}

extern "C" int rafd_get_kernel_times(rafd_room *r, rafd_kernel_times *t)
{
    if (!r || !t) return set_err(RAFD_E_INVAL, "bad arguments");
    CK(cudaSetDevice(r->device));
    resolve_events(r);
    t->volume_ms = r->kt.volume_ms;
    t->boundary_ms = r->kt.boundary_ms;
    t->other_ms = r->kt.other_ms;
    t->volume_launches = r->kt.volume_n;
    t->boundary_launches = r->kt.boundary_n;
    t->other_launches = r->kt.other_n;
    t->shell_ms = r->kt.shell_ms;
    t->shell_launches = r->kt.shell_n;
    return RAFD_OK;
}

extern "C" int64_t rafd_launch_count(rafd_room *r) { return r ? r->launches : 0; }

// ------------------------------------------------------------------ temporal blocking
// Transactional: the second buffer pair and both new plans are built aside and
// swapped in only when every step succeeded; on failure the room is left
// exactly as it was (its single-step plan, graphs and buffers untouched).
template <typename T> static int enable_twostep_t(rafd_room *r)
{
    if (r->tbplan) {
        CK(cudaStreamSynchronize(r->stream));
        return RAFD_OK;
    }
    const size_t fb = (size_t)r->g.total * sizeof(T) + 64;
    void *nu[4] = {r->u[0], r->u[1], r->u[2], r->u[3]};
    bool fresh[4] = {false, false, false, false};
    void *vp = nullptr, *tp = nullptr;
    int64_t nsh = 0;
    cudaError_t e = cudaSuccess;
    int rc = RAFD_OK;
    auto undo = [&]() {
        cudaStreamSynchronize(r->stream);
        if (tp) twostep_plan_destroy(tp);
        if (vp) volume_plan_destroy(vp);
        for (int k = 2; k < 4; k++)
            if (fresh[k]) {
                dfree(r, nu[k]);
                r->device_bytes -= (int64_t)fb + 64;
            }
    };
    PhaseTrace tr("rafd_set_temporal_blocking(2)");
    {
        // the second pair is zeroed on the side stream while the plans are built
        SideWork zero_u(r->stream, r->cap_stream);
        for (int k = 2; k < 4 && rc == RAFD_OK; k++)
            if (!nu[k]) {
                if ((rc = dmalloc(r, &nu[k], fb)) == RAFD_OK) {
                    fresh[k] = true;
                    e = cudaMemsetAsync(nu[k], 0, fb, r->cap_stream);
                    if (e != cudaSuccess) rc = -1;
                }
            }
        zero_u.done();
        tr.mark(r->stream, "alloc u[2..3]");
        // the single-step kernel needs TMA maps of the second pair too
        if (rc == RAFD_OK && e == cudaSuccess) e = volume_plan_create<T>(r->g, nu, r->K_alloc, r->nsm, &vp);
        // (the occupancy table is taken over from the current plan at the commit below)
        tr.mark(r->stream, "volume plan");
        if (rc == RAFD_OK && e == cudaSuccess)
            e = twostep_plan_create<T>(r->g, nu, r->K_alloc, r->K, r->idx64, r->nsm, r->stream, &tp, &nsh);
        tr.mark(r->stream, "two-step plan + shell list");
    }  // the main stream waits for the zeroing here (before any use, synchronisation or undo)
    Ctl<T> c;
    if (rc == RAFD_OK && e == cudaSuccess) {
        if ((rc = pull_ctl<T>(r, c)) == RAFD_OK) e = twostep_set_source(tp, c.src_pos, r->g);
    }
    if (rc == RAFD_OK && e == cudaSuccess) e = cudaStreamSynchronize(r->stream);
    if (rc != RAFD_OK || e != cudaSuccess) {
        undo();
        if (rc != RAFD_OK && rc != -1) return rc;
        cudaGetLastError();
        return set_err(e == cudaErrorMemoryAllocation ? RAFD_E_NOMEM : RAFD_E_CUDA,
                       "enabling temporal blocking: %s", cudaGetErrorString(e));
    }
    // commit: the cached graphs captured the old plan's arguments
    free_graphs(r);
    volume_plan_adopt_occupancy(vp, r->vplan);
    volume_plan_destroy(r->vplan);
    r->vplan = vp;
    r->tbplan = tp;
    r->n_shell = nsh;
    // the fused shell + boundary pass needs the list's node entries to be the
    // room's nodes (always, for a whole room); RAFD_SHELL_BND=0 keeps two passes
    {
        const char *sb = getenv("RAFD_SHELL_BND");
        r->shell_bnd = r->nb > 0 && r->scheme == 0 && twostep_shell_nodes(tp) == r->nb && !(sb && strcmp(sb, "0") == 0);
    }
    r->device_bytes += r->n_shell * (r->idx64 ? 8 : 4) + 56;
    for (int k = 2; k < 4; k++) r->u[k] = nu[k];
    return RAFD_OK;
}

extern "C" int rafd_set_temporal_blocking(rafd_room *r, int32_t steps_per_sweep)
{
    if (!r || (steps_per_sweep != 1 && steps_per_sweep != 2))
        return set_err(RAFD_E_INVAL, "steps_per_sweep must be 1 or 2");
    CK(cudaSetDevice(r->device));
    if (steps_per_sweep == r->tb) return RAFD_OK;
    CK(cudaStreamSynchronize(r->stream));
    if (steps_per_sweep == 2) {
        if (r->ipc && ipc_peer_buffers(r->ipc) < 4)
            return set_err(RAFD_E_STATE, "IPC slabs enable temporal blocking before rafd_ipc_handle (the neighbours "
                                         "exported two field buffers)");
        if (r->scheme != 0 || r->fused)
            return set_err(RAFD_E_STATE, "temporal blocking runs the two-kernel scheme (not fused, not Listing 1/6)");
        if (!r->vplan) return set_err(RAFD_E_STATE, "temporal blocking needs the TMA volume kernel (not v0)");
        int rc = r->prec == 32 ? enable_twostep_t<float>(r) : enable_twostep_t<double>(r);
        if (rc) return rc;
    }
    free_graphs(r);  // the step sequence changed
    r->tb = steps_per_sweep;
    return RAFD_OK;
}

// ------------------------------------------------------------------ host-only helpers
extern "C" int rafd_slab_plan(int32_t nx, int32_t ny, int32_t nz, const uint8_t *mask, int32_t precision,
                              int32_t n_branches, int32_t nranks, int32_t *z_begin, int32_t *z_end)
{
    if (!mask || !z_begin || !z_end || nx < 1 || ny < 1 || nz < 1 || nranks < 1 || nranks > nz)
        return set_err(RAFD_E_INVAL, "bad slab-plan arguments (need 1 <= nranks <= nz)");
    if (precision != 32 && precision != 64) return set_err(RAFD_E_INVAL, "precision must be 32 or 64");
    const int64_t s = precision / 8;
    const int64_t nxny = (int64_t)nx * ny;
    // per-plane cost c(z) = N_mask(z) + 3s N_in(z) + (6 + 3s + 4s MB) Nb(z)
    std::vector<double> cost((size_t)nz);
    auto in = [&](int64_t x, int64_t y, int64_t z) -> int {
        if (x < 0 || y < 0 || z < 0 || x >= nx || y >= ny || z >= nz) return 0;
        return mask[(z * ny + y) * nx + x] ? 1 : 0;
    };
    for (int64_t z = 0; z < nz; z++) {
        int64_t nin = 0, nb = 0;
        for (int64_t y = 0; y < ny; y++)
            for (int64_t x = 0; x < nx; x++) {
                if (!in(x, y, z)) continue;
                const int k = in(x - 1, y, z) + in(x + 1, y, z) + in(x, y - 1, z) + in(x, y + 1, z) +
                              in(x, y, z - 1) + in(x, y, z + 1);
                if (k > 0) nin++;
                if (k > 0 && k < 6) nb++;
            }
        cost[(size_t)z] = (double)nxny + 3.0 * s * nin + (6.0 + 3.0 * s + 4.0 * s * n_branches) * nb;
    }
    std::vector<double> pre((size_t)nz + 1, 0.0);
    for (int z = 0; z < nz; z++) pre[(size_t)z + 1] = pre[(size_t)z] + cost[(size_t)z];
    const double tot = pre[(size_t)nz];
    int prev = 0;
    for (int k = 0; k < nranks; k++) {
        z_begin[k] = prev;
        int e;
        if (k == nranks - 1) {
            e = nz;
        } else {
            const double target = tot * (k + 1) / nranks;
            e = (int)(std::lower_bound(pre.begin(), pre.end(), target) - pre.begin());
            // choose the closer cut of the two around the target
            if (e > 0 && fabs(pre[(size_t)e - 1] - target) <= fabs(pre[(size_t)e] - target)) e -= 1;
            e = std::max(e, prev + 1);
            e = std::min(e, nz - (nranks - 1 - k));
        }
        z_end[k] = e;
        prev = e;
    }
    return RAFD_OK;
}

extern "C" int rafd_nccl_unique_id(uint8_t *id128)
{
    if (!id128) return set_err(RAFD_E_INVAL, "null id");
    int rc = halo_unique_id(id128);
    if (rc) return set_err(rc, "%s", halo_last_error());
    return RAFD_OK;
}

extern "C" const char *rafd_last_error(void) { return g_err.c_str(); }

extern "C" const char *rafd_strerror(int code)
{
    switch (code) {
        case RAFD_OK: return "ok";
        case RAFD_E_INVAL: return "invalid argument";
        case RAFD_E_UNSTABLE: return "unstable Courant number (lambda^2 > 1/3)";
        case RAFD_E_NONPASSIVE: return "non-passive boundary material";
        case RAFD_E_OUTSIDE: return "position outside the room";
        case RAFD_E_MATERIAL: return "material id out of range";
        case RAFD_E_NOMEM: return "out of memory";
        case RAFD_E_CUDA: return "CUDA error";
        case RAFD_E_NCCL: return "NCCL error";
        case RAFD_E_STATE: return "invalid state";
        default: return "unknown error";
    }
}

extern "C" int rafd_version(void) { return RAFD_VERSION; }
