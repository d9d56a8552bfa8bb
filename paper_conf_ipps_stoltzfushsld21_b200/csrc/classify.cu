// classify.cu -- voxel classification (row a1 of SURVEY §8(a)), on the device.
//
// PAPER.md:306-323 (Sec. II-B): "nbrs stores the number of neighbors lying
// within the boundary, which is pre-calculated for a given shape.  A value of
// zero is used for points outside."  PAPER.md:390-393: boundaryIndices = the
// indices of the points at the boundary (0 < K < 6, Listing 1 rule,
// PAPER.md:280-291).  PAPER.md:411-412: material per boundary point.
// Readings R2-R4: the library pads the mask with one outside
// layer, isolated inside voxels get K = 0, the boundary list is in ascending
// canonical order, material ids are sampled from the per-voxel matmap.
//
// Passes (all on the K grid itself, no extra full-size buffer):
//   scatter_mask : K[p] = 0x80 where the mask is set (chunks of planes; the
//                  slab's two ghost planes included)
//   count_k      : K[p] = 0x80 | (# of 6 face neighbours with bit 7) for owned
//                  inside voxels (bit 7 is never changed, so concurrent
//                  neighbour reads are consistent)
//   finish_k     : K[p] &= 0x7f on owned planes, histogram (ghost planes keep
//                  their 0x80 flags)
//   row_counts   : boundary nodes per (z, y) row
//   exclusive scan (CUB) -> row offsets
//   compact      : per row, a block scan writes the nodes in ascending x
//   gather_mat   : matb[i] = matmap[bidx[i]], flagging ids >= M
#include <cub/block/block_reduce.cuh>
#include <cub/block/block_scan.cuh>
#include <cub/device/device_scan.cuh>

#include "internal.cuh"

namespace rafd {

static __device__ __forceinline__ int64_t pidx(const Grid &g, int64_t zp, int64_t y, int64_t x)
{
    return zp * g.plane + (y + 1) * g.pitch + g.xo + x;
}

// mask_chunk holds nzc planes starting at local padded plane zp0.
__global__ void k_scatter_mask(Grid g, const uint8_t *__restrict__ mask, int zp0, int nzc,
                               uint8_t *__restrict__ K)
{
    const int64_t n = (int64_t)nzc * g.ny * g.nx;
    for (int64_t c = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; c < n;
         c += (int64_t)gridDim.x * blockDim.x) {
        const int64_t x = c % g.nx;
        const int64_t r = c / g.nx;
        const int64_t y = r % g.ny;
        const int64_t z = r / g.ny;
        K[pidx(g, zp0 + z, y, x)] = mask[c] ? 0x80 : 0;
    }
}

__global__ void k_count_k(Grid g, uint8_t *__restrict__ K)
{
    const int x = blockIdx.x * blockDim.x + threadIdx.x;
    const int y = blockIdx.y;
    const int zp = blockIdx.z + 1;
    if (x >= g.nx) return;
    const int64_t i = pidx(g, zp, y, x);
    const uint8_t v = K[i];
    if (!(v & 0x80)) return;
    const int k = (K[i - 1] >> 7) + (K[i + 1] >> 7) + (K[i - g.pitch] >> 7) + (K[i + g.pitch] >> 7) +
                  (K[i - g.plane] >> 7) + (K[i + g.plane] >> 7);
    K[i] = (uint8_t)(0x80 | k);
}

__global__ void k_finish_k(Grid g, uint8_t *__restrict__ K, unsigned long long *hist)
{
    __shared__ unsigned int h[8];
    if (threadIdx.x < 8) h[threadIdx.x] = 0;
    __syncthreads();
    const int64_t n = (int64_t)g.lnz * g.ny * g.nx;
    for (int64_t c = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; c < n;
         c += (int64_t)gridDim.x * blockDim.x) {
        const int64_t x = c % g.nx;
        const int64_t r = c / g.nx;
        const int64_t y = r % g.ny;
        const int64_t z = r / g.ny;
        const int64_t i = pidx(g, z + 1, y, x);
        const uint8_t v = K[i];
        if (v & 0x80) {
            const int k = v & 0x7f;
            K[i] = (uint8_t)k;
            atomicAdd(&h[k], 1u);
        }
    }
    __syncthreads();
    if (threadIdx.x < 8 && h[threadIdx.x]) atomicAdd(&hist[threadIdx.x], (unsigned long long)h[threadIdx.x]);
}

__global__ void k_row_counts(Grid g, const uint8_t *__restrict__ K, int64_t *__restrict__ counts)
{
    using BR = cub::BlockReduce<int, 256>;
    __shared__ typename BR::TempStorage tmp;
    const int64_t row = blockIdx.x;  // = zl*ny + y
    const int64_t y = row % g.ny, zl = row / g.ny;
    const int64_t base = pidx(g, zl + 1, y, 0);
    int c = 0;
    for (int x = threadIdx.x; x < g.nx; x += 256) {
        const int k = K[base + x];
        c += (k > 0 && k < 6);
    }
    c = BR(tmp).Sum(c);
    if (threadIdx.x == 0) counts[row] = c;
}

template <typename IdxT>
__global__ void k_compact(Grid g, const uint8_t *__restrict__ K, const int64_t *__restrict__ row_off,
                          int64_t zglob0, int32_t ny_glob, int32_t nx_glob, IdxT *__restrict__ bpos,
                          int64_t *__restrict__ bidx, uint8_t *__restrict__ Kb)
{
    using BS = cub::BlockScan<int, 256>;
    __shared__ typename BS::TempStorage tmp;
    const int64_t row = blockIdx.x;
    const int64_t y = row % g.ny, zl = row / g.ny;
    const int64_t base = pidx(g, zl + 1, y, 0);
    int64_t out = row_off[row];
    for (int x0 = 0; x0 < g.nx; x0 += 256) {
        const int x = x0 + threadIdx.x;
        int k = (x < g.nx) ? K[base + x] : 0;
        const int f = (k > 0 && k < 6);
        int pre, tot;
        BS(tmp).ExclusiveSum(f, pre, tot);
        if (f) {
            const int64_t o = out + pre;
            bpos[o] = (IdxT)(base + x);
            bidx[o] = ((zglob0 + zl) * ny_glob + y) * nx_glob + x;
            Kb[o] = (uint8_t)k;
        }
        out += tot;
        __syncthreads();
    }
}

__global__ void k_gather_mat(const uint8_t *__restrict__ mm, int64_t canon0,
                             const int64_t *__restrict__ bidx, int64_t i_lo, int64_t i_hi,
                             uint8_t *__restrict__ matb, int M, unsigned int *bad)
{
    for (int64_t i = i_lo + (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < i_hi;
         i += (int64_t)gridDim.x * blockDim.x) {
        const uint8_t m = mm ? mm[bidx[i] - canon0] : 0;
        matb[i] = m;
        if (m >= M) atomicOr(bad, 1u);
    }
}

static unsigned grid_for(int64_t n, int threads = 256)
{
    int64_t b = (n + threads - 1) / threads;
    if (b > 148 * 32) b = 148 * 32;
    if (b < 1) b = 1;
    return (unsigned)b;
}

cudaError_t launch_scatter_mask(const Grid &g, const uint8_t *mask_chunk, int zp0, int nzc,
                                uint8_t *K, cudaStream_t s)
{
    const int64_t n = (int64_t)nzc * g.ny * g.nx;
    if (n == 0) return cudaSuccess;
    k_scatter_mask<<<grid_for(n), 256, 0, s>>>(g, mask_chunk, zp0, nzc, K);
    return cudaGetLastError();
}

cudaError_t launch_count_k(const Grid &g, uint8_t *K, cudaStream_t s)
{
    dim3 grid((g.nx + 255) / 256, g.ny, g.lnz);
    k_count_k<<<grid, 256, 0, s>>>(g, K);
    return cudaGetLastError();
}

cudaError_t launch_finish_k(const Grid &g, uint8_t *K, unsigned long long *hist8, cudaStream_t s)
{
    const int64_t n = (int64_t)g.lnz * g.ny * g.nx;
    k_finish_k<<<grid_for(n), 256, 0, s>>>(g, K, hist8);
    // the two ghost planes keep their 0x80 inside flags: set_state / read use
    // them to keep ghost values, the energy hook for cross-slab edges; no
    // kernel of the step reads K there
    return cudaGetLastError();
}

cudaError_t launch_row_counts64(const Grid &g, const uint8_t *K, int64_t *counts, cudaStream_t s)
{
    const int64_t rows = (int64_t)g.lnz * g.ny;
    if (rows == 0) return cudaSuccess;
    k_row_counts<<<(unsigned)rows, 256, 0, s>>>(g, K, counts);
    return cudaGetLastError();
}

cudaError_t launch_compact(const Grid &g, const uint8_t *K, const int64_t *row_off, int64_t zglob0,
                           int32_t ny_glob, int32_t nx_glob, bool idx64, void *bpos,
                           int64_t *bidx, uint8_t *Kb, cudaStream_t s)
{
    const int64_t rows = (int64_t)g.lnz * g.ny;
    if (rows == 0) return cudaSuccess;
    if (idx64)
        k_compact<int64_t><<<(unsigned)rows, 256, 0, s>>>(g, K, row_off, zglob0, ny_glob, nx_glob,
                                                          (int64_t *)bpos, bidx, Kb);
    else
        k_compact<uint32_t><<<(unsigned)rows, 256, 0, s>>>(g, K, row_off, zglob0, ny_glob, nx_glob,
                                                           (uint32_t *)bpos, bidx, Kb);
    return cudaGetLastError();
}

cudaError_t launch_gather_mat(const uint8_t *matmap_chunk, int64_t canon0, const int64_t *bidx,
                              int64_t i_lo, int64_t i_hi, uint8_t *matb, int M,
                              unsigned int *bad_flag, cudaStream_t s)
{
    if (i_hi <= i_lo) return cudaSuccess;
    k_gather_mat<<<grid_for(i_hi - i_lo), 256, 0, s>>>(matmap_chunk, canon0, bidx, i_lo, i_hi, matb,
                                                       M, bad_flag);
    return cudaGetLastError();
}

cudaError_t exclusive_scan_rows64(const int64_t *counts, int64_t *row_off, int64_t n, void *tmp,
                                  size_t *tmp_bytes, cudaStream_t s)
{
    return cub::DeviceScan::ExclusiveSum(tmp, *tmp_bytes, counts, row_off, (int)n, s);
}

}  // namespace rafd
