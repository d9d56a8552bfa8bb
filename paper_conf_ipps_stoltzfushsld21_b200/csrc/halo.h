// halo.h -- z-slab halo exchange between ranks: after every
// step each rank sends its first / last owned plane to rank-1 / rank+1 and
// receives their edge planes into its two ghost planes.  NCCL point-to-point
// (ncclSend / ncclRecv in one group) on the room's stream; libnccl is loaded
// with dlopen so that single-GPU use never needs it.
#pragma once
#include <cuda_runtime.h>
#include <stddef.h>
#include <stdint.h>

namespace rafd {
struct Halo;
int halo_create(Halo **out, const uint8_t *nccl_id, int rank, int nranks, cudaStream_t s);
void halo_destroy(Halo *h);
// buf: padded field with (lnz+2) planes of plane_bytes each
cudaError_t halo_exchange(Halo *h, void *buf, size_t plane_bytes, int lnz, cudaStream_t s);
int halo_unique_id(uint8_t *id128);
const char *halo_last_error();
}  // namespace rafd

// ---------------------------------------------------------------- IPC transport
// Slabs in different processes (same or peer GPUs): each rank maps its
// neighbours' two field buffers and 16-byte signal words via CUDA IPC, copies
// the neighbours' edge planes into its ghost planes with device-to-device
// copies, and orders everything with GPU-side stream memory operations
// (cuStreamWriteValue64 / cuStreamWaitValue64 on the signal words): no host
// round trip, no NCCL.  Signal word 0 = "edge planes of step n done" (n+1),
// word 1 = "my copies out of my neighbours' buffers for step n done" (n+1).
namespace rafd {
struct HaloIpc;
constexpr int kIpcBlobBytes = 5 * 64 + 32;
// blob of this rank: IPC handles of u[0..3] (u[2], u[3] -- the second pair of
// temporal blocking -- may be null: nbuf = 2) and sig, then (magic, device,
// lnz, pitch, nbuf)
int ipc_make_blob(void *const u[4], int64_t *sig, int device, int lnz, uint32_t pitch, uint8_t *blob);
// number of field buffers every connected neighbour exported (2 or 4)
int ipc_peer_buffers(const HaloIpc *h);
int ipc_open(HaloIpc **out, const uint8_t *lower, const uint8_t *upper, uint32_t pitch);
void ipc_close(HaloIpc *h);
// per-step pieces (stream-ordered)
cudaError_t ipc_signal(int64_t *addr, int64_t value, cudaStream_t s);
cudaError_t ipc_wait_peers(HaloIpc *h, int word, int64_t value, cudaStream_t s);
cudaError_t ipc_pull(HaloIpc *h, int buf, void *mine, size_t plane_bytes, int lnz, cudaStream_t s);
void ipc_mirror_deltas(HaloIpc *h, int buf, const void *mine, size_t plane_bytes, int lnz, int64_t *d_lo,
                       int64_t *d_hi);
}  // namespace rafd
