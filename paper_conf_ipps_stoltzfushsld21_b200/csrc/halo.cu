// halo.cu -- NCCL halo exchange for z-slab decomposition (see halo.h).
#include <dlfcn.h>
#include <stdio.h>
#include <string.h>

#include <string>
#include <algorithm>

#include "../../include/rafd.h"
#include "halo.h"

namespace rafd {

// Minimal NCCL ABI (stable since NCCL 2.0): opaque communicator, 128-byte id.
typedef struct ncclComm *ncclComm_t;
typedef struct {
    char internal[128];
} ncclUniqueId;
typedef int ncclResult_t;
static const int ncclInt8 = 0;

struct NcclApi {
    void *lib = nullptr;
    ncclResult_t (*GetUniqueId)(ncclUniqueId *) = nullptr;
    ncclResult_t (*CommInitRank)(ncclComm_t *, int, ncclUniqueId, int) = nullptr;
    ncclResult_t (*CommDestroy)(ncclComm_t) = nullptr;
    ncclResult_t (*Send)(const void *, size_t, int, int, ncclComm_t, cudaStream_t) = nullptr;
    ncclResult_t (*Recv)(void *, size_t, int, int, ncclComm_t, cudaStream_t) = nullptr;
    ncclResult_t (*GroupStart)() = nullptr;
    ncclResult_t (*GroupEnd)() = nullptr;
    const char *(*GetErrorString)(ncclResult_t) = nullptr;
    ncclResult_t (*CommGetAsyncError)(ncclComm_t, ncclResult_t *) = nullptr;  // NCCL >= 2.4 (optional)
};
static const int ncclInProgress = 7;

static thread_local std::string h_err;
const char *halo_last_error() { return h_err.c_str(); }

static NcclApi *api()
{
    static NcclApi a;
    static bool tried = false;
    if (tried) return a.lib ? &a : nullptr;
    tried = true;
    const char *names[] = {"libnccl.so.2", "libnccl.so"};
    for (const char *n : names) {
        a.lib = dlopen(n, RTLD_NOW | RTLD_GLOBAL);
        if (a.lib) break;
    }
    if (!a.lib) {
        h_err = std::string("cannot dlopen libnccl.so.2: ") + dlerror();
        return nullptr;
    }
#define SYM(f, n)                                               \
    *(void **)(&a.f) = dlsym(a.lib, n);                         \
    if (!a.f) {                                                 \
        h_err = std::string("libnccl lacks ") + n;              \
        a.lib = nullptr;                                        \
        return nullptr;                                         \
    }
    SYM(GetUniqueId, "ncclGetUniqueId")
    SYM(CommInitRank, "ncclCommInitRank")
    SYM(CommDestroy, "ncclCommDestroy")
    SYM(Send, "ncclSend")
    SYM(Recv, "ncclRecv")
    SYM(GroupStart, "ncclGroupStart")
    SYM(GroupEnd, "ncclGroupEnd")
    SYM(GetErrorString, "ncclGetErrorString")
#undef SYM
    *(void **)(&a.CommGetAsyncError) = dlsym(a.lib, "ncclCommGetAsyncError");
    return &a;
}

struct Halo {
    ncclComm_t comm = nullptr;
    int rank = 0, nranks = 1;
};

int halo_unique_id(uint8_t *id128)
{
    NcclApi *a = api();
    if (!a) return RAFD_E_NCCL;
    ncclUniqueId id;
    ncclResult_t r = a->GetUniqueId(&id);
    if (r != 0) {
        h_err = std::string("ncclGetUniqueId: ") + a->GetErrorString(r);
        return RAFD_E_NCCL;
    }
    memcpy(id128, id.internal, 128);
    return RAFD_OK;
}

int halo_create(Halo **out, const uint8_t *nccl_id, int rank, int nranks, cudaStream_t s)
{
    (void)s;
    *out = nullptr;
    if (!nccl_id) {
        h_err = "nranks > 1 needs the 128-byte nccl_id from rafd_nccl_unique_id";
        return RAFD_E_INVAL;
    }
    NcclApi *a = api();
    if (!a) return RAFD_E_NCCL;
    ncclUniqueId id;
    memcpy(id.internal, nccl_id, 128);
    Halo *h = new Halo();
    h->rank = rank;
    h->nranks = nranks;
    ncclResult_t r = a->CommInitRank(&h->comm, nranks, id, rank);
    if (r != 0) {
        h_err = std::string("ncclCommInitRank: ") + a->GetErrorString(r);
        delete h;
        return RAFD_E_NCCL;
    }
    *out = h;
    return RAFD_OK;
}

void halo_destroy(Halo *h)
{
    if (!h) return;
    NcclApi *a = api();
    if (a && h->comm) a->CommDestroy(h->comm);
    delete h;
}

cudaError_t halo_exchange(Halo *h, void *buf, size_t plane_bytes, int lnz, cudaStream_t s)
{
    NcclApi *a = api();
    if (!a) return cudaErrorUnknown;
    char *b = (char *)buf;
    ncclResult_t r = a->GroupStart();
    if (h->rank > 0) {
        if (!r) r = a->Send(b + plane_bytes, plane_bytes, ncclInt8, h->rank - 1, h->comm, s);
        if (!r) r = a->Recv(b, plane_bytes, ncclInt8, h->rank - 1, h->comm, s);
    }
    if (h->rank < h->nranks - 1) {
        if (!r) r = a->Send(b + (size_t)lnz * plane_bytes, plane_bytes, ncclInt8, h->rank + 1, h->comm, s);
        if (!r) r = a->Recv(b + (size_t)(lnz + 1) * plane_bytes, plane_bytes, ncclInt8, h->rank + 1, h->comm, s);
    }
    ncclResult_t r2 = a->GroupEnd();
    if (r || r2) {
        h_err = std::string("nccl halo exchange: ") + a->GetErrorString(r ? r : r2);
        return cudaErrorUnknown;
    }
    // an asynchronous fault (a peer died, a network error) would otherwise
    // surface only as a hang or wrong ghost planes
    if (a->CommGetAsyncError) {
        ncclResult_t ae = 0;
        ncclResult_t q = a->CommGetAsyncError(h->comm, &ae);
        if (q != 0 || (ae != 0 && ae != ncclInProgress)) {
            h_err = std::string("nccl asynchronous error: ") + a->GetErrorString(q ? q : ae);
            return cudaErrorUnknown;
        }
    }
    return cudaGetLastError();
}

}  // namespace rafd

// ================================================================ IPC transport
#include <cudaTypedefs.h>

namespace rafd {

struct IpcPeer {
    void *u[4] = {nullptr, nullptr, nullptr, nullptr};
    int nbuf = 0;
    int64_t *sig = nullptr;
    bool open = false;
    int lnz = 0;
    uint32_t pitch = 0;
};

struct HaloIpc {
    IpcPeer lo, hi;
};

static const uint32_t kMagic = 0x52414644u;  // "RAFD"

struct StreamMemOps {
    PFN_cuStreamWaitValue32_v2 wait = nullptr;
    PFN_cuStreamWriteValue32_v2 write = nullptr;
    bool ok = false;
};

static StreamMemOps &memops()
{
    static StreamMemOps m;
    static bool tried = false;
    if (!tried) {
        tried = true;
        cudaDriverEntryPointQueryResult q;
        void *p = nullptr;
        if (cudaGetDriverEntryPoint("cuStreamWaitValue32", &p, cudaEnableDefault, &q) == cudaSuccess &&
            q == cudaDriverEntryPointSuccess)
            m.wait = (PFN_cuStreamWaitValue32_v2)p;
        p = nullptr;
        if (cudaGetDriverEntryPoint("cuStreamWriteValue32", &p, cudaEnableDefault, &q) == cudaSuccess &&
            q == cudaDriverEntryPointSuccess)
            m.write = (PFN_cuStreamWriteValue32_v2)p;
        m.ok = m.wait && m.write;
        if (!m.ok) h_err = "cuStreamWaitValue32/cuStreamWriteValue32 unavailable";
    }
    return m;
}

int ipc_make_blob(void *const u[4], int64_t *sig, int device, int lnz, uint32_t pitch, uint8_t *blob)
{
    memset(blob, 0, kIpcBlobBytes);
    const int nbuf = (u[2] && u[3]) ? 4 : 2;
    void *p[5] = {u[0], u[1], nbuf == 4 ? u[2] : nullptr, nbuf == 4 ? u[3] : nullptr, sig};
    for (int k = 0; k < 5; k++) {
        if (!p[k]) continue;
        cudaIpcMemHandle_t h;
        cudaError_t e = cudaIpcGetMemHandle(&h, p[k]);
        if (e != cudaSuccess) {
            h_err = std::string("cudaIpcGetMemHandle: ") + cudaGetErrorString(e);
            return RAFD_E_CUDA;
        }
        memcpy(blob + 64 * k, &h, 64);
    }
    uint32_t tail[8] = {kMagic, (uint32_t)device, (uint32_t)lnz, pitch, (uint32_t)nbuf, 0, 0, 0};
    memcpy(blob + 320, tail, 32);
    return RAFD_OK;
}

static int open_peer(IpcPeer &pe, const uint8_t *blob)
{
    uint32_t tail[8];
    memcpy(tail, blob + 320, 32);
    if (tail[0] != kMagic) {
        h_err = "not a rafd IPC blob";
        return RAFD_E_INVAL;
    }
    pe.lnz = (int)tail[2];
    pe.pitch = tail[3];
    pe.nbuf = (int)tail[4];
    void **dst[5] = {&pe.u[0], &pe.u[1], &pe.u[2], &pe.u[3], (void **)&pe.sig};
    for (int k = 0; k < 5; k++) {
        if (k >= pe.nbuf && k < 4) continue;
        cudaIpcMemHandle_t h;
        memcpy(&h, blob + 64 * k, 64);
        cudaError_t e = cudaIpcOpenMemHandle(dst[k], h, cudaIpcMemLazyEnablePeerAccess);
        if (e != cudaSuccess) {
            h_err = std::string("cudaIpcOpenMemHandle: ") + cudaGetErrorString(e);
            return RAFD_E_CUDA;
        }
    }
    pe.open = true;
    return RAFD_OK;
}

int ipc_peer_buffers(const HaloIpc *h)
{
    int n = 4;
    for (const IpcPeer *pe : {&h->lo, &h->hi})
        if (pe->open) n = std::min(n, pe->nbuf);
    return n;
}

int ipc_open(HaloIpc **out, const uint8_t *lower, const uint8_t *upper, uint32_t pitch)
{
    *out = nullptr;
    for (const uint8_t *b : {lower, upper}) {
        if (!b) continue;
        uint32_t tail[8];
        memcpy(tail, b + 320, 32);
        if (tail[0] != kMagic || tail[3] != pitch) {
            h_err = "IPC blob is not a slab of the same room (magic / pitch mismatch)";
            return RAFD_E_INVAL;
        }
    }
    if (!memops().ok) return RAFD_E_CUDA;
    HaloIpc *h = new HaloIpc();
    int rc = RAFD_OK;
    if (lower) rc = open_peer(h->lo, lower);
    if (!rc && upper) rc = open_peer(h->hi, upper);
    if (rc) {
        ipc_close(h);
        return rc;
    }
    *out = h;
    return RAFD_OK;
}

void ipc_close(HaloIpc *h)
{
    if (!h) return;
    for (IpcPeer *pe : {&h->lo, &h->hi}) {
        if (!pe->open) continue;
        for (int k = 0; k < 4; k++)
            if (pe->u[k]) cudaIpcCloseMemHandle(pe->u[k]);
        if (pe->sig) cudaIpcCloseMemHandle(pe->sig);
    }
    delete h;
}

// 32-bit stream memory operations (64-bit ones need an optional device
// capability); step counters stay far below 2^31.
cudaError_t ipc_signal(int64_t *addr, int64_t value, cudaStream_t s)
{
    // default flags: ordered after prior work in the stream, with a memory barrier
    CUresult r = memops().write((CUstream)s, (CUdeviceptr)addr, (cuuint32_t)value, CU_STREAM_WRITE_VALUE_DEFAULT);
    if (r != CUDA_SUCCESS) {
        h_err = "cuStreamWriteValue32 failed (CUresult " + std::to_string((int)r) + ")";
        return cudaErrorUnknown;
    }
    return cudaSuccess;
}

cudaError_t ipc_wait_peers(HaloIpc *h, int word, int64_t value, cudaStream_t s)
{
    for (IpcPeer *pe : {&h->lo, &h->hi}) {
        if (!pe->open) continue;
        CUresult r = memops().wait((CUstream)s, (CUdeviceptr)(pe->sig + word), (cuuint32_t)value,
                                   CU_STREAM_WAIT_VALUE_GEQ);
        if (r != CUDA_SUCCESS) {
            h_err = "cuStreamWaitValue32 failed (CUresult " + std::to_string((int)r) + ")";
            return cudaErrorUnknown;
        }
    }
    return cudaSuccess;
}

// halo push (device-initiated): byte offsets that take an address in my
// buffer `buf` to the same voxel in a neighbour's ghost plane of its buffer
// `buf` -- my first owned plane (padded 1) -> the lower neighbour's top ghost
// (its padded lnz_lo + 1); my last (padded lnz) -> the upper neighbour's
// bottom ghost (padded 0).  0 where there is no neighbour.
void ipc_mirror_deltas(HaloIpc *h, int buf, const void *mine, size_t plane_bytes, int lnz, int64_t *d_lo,
                       int64_t *d_hi)
{
    *d_lo = *d_hi = 0;
    if (h->lo.open)
        *d_lo = (int64_t)((uintptr_t)h->lo.u[buf] - (uintptr_t)mine) + (int64_t)h->lo.lnz * (int64_t)plane_bytes;
    if (h->hi.open)
        *d_hi = (int64_t)((uintptr_t)h->hi.u[buf] - (uintptr_t)mine) - (int64_t)lnz * (int64_t)plane_bytes;
}

// ghost planes of my buffer `buf` <- the neighbours' edge planes of their buffer `buf`
// (all slabs step in lock-step, so they use the same buffer parity)
cudaError_t ipc_pull(HaloIpc *h, int buf, void *mine, size_t plane_bytes, int lnz, cudaStream_t s)
{
    char *m = (char *)mine;
    cudaError_t e = cudaSuccess;
    if (h->lo.open)
        e = cudaMemcpyAsync(m, (const char *)h->lo.u[buf] + (size_t)h->lo.lnz * plane_bytes, plane_bytes,
                            cudaMemcpyDeviceToDevice, s);
    if (e == cudaSuccess && h->hi.open)
        e = cudaMemcpyAsync(m + (size_t)(lnz + 1) * plane_bytes, (const char *)h->hi.u[buf] + plane_bytes,
                            plane_bytes, cudaMemcpyDeviceToDevice, s);
    return e;
}

}  // namespace rafd
