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
