// halo.cu -- NCCL halo exchange for z-slab decomposition (see halo.h).
#include <dlfcn.h>
#include <stdio.h>
#include <string.h>

#include <string>

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
};

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
    return cudaGetLastError();
}

}  // namespace rafd
