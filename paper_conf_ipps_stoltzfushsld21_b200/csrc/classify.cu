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
// Passes (all on the K grid itself, no extra full-size buffer; bytes are
// processed as SIMD lanes of 32-bit words, 16 voxels per thread and step):
//   scatter_mask : K[p] = 0x80 where the mask is set (chunks of planes; the
//                  slab's two ghost planes included)
//   count_k      : K[p] = 0x80 | (# of 6 face neighbours with bit 7) for owned
//                  inside voxels (bit 7 is never changed, so concurrent
//                  neighbour reads are consistent)
//   finish_k     : K[p] &= 0x7f on owned planes, histogram (ghost planes keep
//                  their 0x80 flags)
//   row_counts   : boundary nodes per (z, y) row (one warp per row)
//   exclusive scan (CUB) -> row offsets
//   compact      : per row, a warp scan writes the nodes in ascending x
//   gather_mat   : matb[i] = matmap[bidx[i]], flagging ids >= M
// The shell list of the two-step kernel (twostep.cu) uses the same row count /
// compaction with its own selection.
#include <cub/device/device_scan.cuh>

#include "internal.cuh"

namespace rafd {

static __device__ __forceinline__ int64_t pidx(const Grid &g, int64_t zp, int64_t y, int64_t x)
{
    return zp * g.plane + (y + 1) * g.pitch + g.xo + x;
}

// ---- bytes as SIMD lanes (four voxels per 32-bit word, sixteen per uint4).
// Element x = 0 of every K row is 16-byte aligned (k_shift, internal.cuh), so a
// row is read as 16-byte chunks; bytes past nx are the zero halo / padding.
// Each helper returns 0x80 in the bytes where the predicate holds, exactly
// (no carry or borrow crosses a byte).
namespace swar {
static __device__ __forceinline__ uint32_t zero(uint32_t x)  // byte == 0
{
    const uint32_t t = (x & 0x7F7F7F7Fu) + 0x7F7F7F7Fu;
    return ~(t | x | 0x7F7F7F7Fu);
}
static __device__ __forceinline__ uint32_t lt(uint32_t x, uint32_t k4)  // byte < k (k <= 0x80), k4 = k * 0x01010101
{
    const uint32_t t = (x | 0x80808080u) - k4;
    return ~(t | x) & 0x80808080u;
}
static __device__ __forceinline__ uint32_t bnd(uint32_t x) { return lt(x, 0x06060606u) & ~zero(x) & 0x80808080u; }
// the x-1 / x+1 neighbour bytes of word w (prev: the word before, next: after)
static __device__ __forceinline__ uint32_t xm(uint32_t w, uint32_t prev) { return (w << 8) | (prev >> 24); }
static __device__ __forceinline__ uint32_t xp(uint32_t w, uint32_t next) { return (w >> 8) | (next << 24); }
static __device__ __forceinline__ uint32_t w4(const uint4 &v, int i) { return i == 0 ? v.x : i == 1 ? v.y : i == 2 ? v.z : v.w; }
}  // namespace swar

// mask_chunk holds nzc planes starting at local padded plane zp0: one warp per
// row, K = 0x80 where the mask is set (16 bytes per lane and step).
__global__ void k_scatter_mask(Grid g, const uint8_t *__restrict__ mask, int zp0, int nzc,
                               uint8_t *__restrict__ K)
{
    const int lane = threadIdx.x & 31;
    const int64_t rows = (int64_t)nzc * g.ny, nch = (g.nx + 15) / 16;
    const bool vec = (g.nx & 15) == 0 && ((uintptr_t)mask & 15) == 0;
    for (int64_t row = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; row < rows;
         row += ((int64_t)gridDim.x * blockDim.x) >> 5) {
        const int64_t y = row % g.ny, z = row / g.ny;
        const uint8_t *m = mask + row * g.nx;
        uint8_t *k = K + pidx(g, zp0 + z, y, 0);
        for (int64_t c = lane; c < nch; c += 32) {
            uint32_t w[4];
            if (vec) {
                const uint4 v = *(const uint4 *)(m + 16 * c);
                w[0] = v.x; w[1] = v.y; w[2] = v.z; w[3] = v.w;
            } else {
#pragma unroll
                for (int i = 0; i < 4; i++) {
                    uint32_t a = 0;
#pragma unroll
                    for (int b = 0; b < 4; b++) {
                        const int64_t x = 16 * c + 4 * i + b;
                        if (x < g.nx) a |= (uint32_t)m[x] << (8 * b);
                    }
                    w[i] = a;
                }
            }
            uint4 o;
            o.x = ~swar::zero(w[0]) & 0x80808080u;
            o.y = ~swar::zero(w[1]) & 0x80808080u;
            o.z = ~swar::zero(w[2]) & 0x80808080u;
            o.w = ~swar::zero(w[3]) & 0x80808080u;
            *(uint4 *)(k + 16 * c) = o;
        }
    }
}

// K = 0x80 | (# of the six face neighbours with bit 7) for owned inside voxels;
// 16 voxels per item.  Bit 7 never changes, so the neighbour words other items
// rewrite concurrently are read consistently.
__global__ void k_count_k(Grid g, uint8_t *__restrict__ K)
{
    const int64_t nch = (g.nx + 15) / 16, items = (int64_t)g.lnz * g.ny * nch;
    for (int64_t it = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; it < items;
         it += (int64_t)gridDim.x * blockDim.x) {
        const int64_t c = it % nch, row = it / nch;
        const int64_t y = row % g.ny, zl = row / g.ny;
        uint8_t *p = K + pidx(g, zl + 1, y, 16 * c);
        const uint4 w = *(const uint4 *)p;
        if ((w.x | w.y | w.z | w.w) == 0) continue;  // no inside voxel here
        const uint4 ym = *(const uint4 *)(p - g.pitch), yp = *(const uint4 *)(p + g.pitch);
        const uint4 zm = *(const uint4 *)(p - g.plane), zp = *(const uint4 *)(p + g.plane);
        const uint32_t before = (uint32_t)p[-1] << 24, after = p[16];
        uint4 o;
#pragma unroll
        for (int i = 0; i < 4; i++) {
            const uint32_t wi = swar::w4(w, i);
            const uint32_t prev = i == 0 ? before : swar::w4(w, i - 1);
            const uint32_t next = i == 3 ? after : swar::w4(w, i + 1);
            const uint32_t f = 0x01010101u;
            const uint32_t cnt = ((swar::xm(wi, prev) >> 7) & f) + ((swar::xp(wi, next) >> 7) & f) +
                                 ((swar::w4(ym, i) >> 7) & f) + ((swar::w4(yp, i) >> 7) & f) +
                                 ((swar::w4(zm, i) >> 7) & f) + ((swar::w4(zp, i) >> 7) & f);
            const uint32_t in = ((wi >> 7) & f) * 0xFFu;  // 0xFF in the inside bytes
            const uint32_t r = (wi & 0x80808080u) | (cnt & in);
            if (i == 0) o.x = r; else if (i == 1) o.y = r; else if (i == 2) o.z = r; else o.w = r;
        }
        *(uint4 *)p = o;
    }
}

// K &= 0x7f on owned planes and the histogram of K over inside voxels (bin 0:
// isolated inside voxels); one warp per row, per-warp bins, one atomic per bin
// and block.
__global__ void k_finish_k(Grid g, uint8_t *__restrict__ K, unsigned long long *hist)
{
    __shared__ unsigned long long h[7];
    if (threadIdx.x < 7) h[threadIdx.x] = 0;
    __syncthreads();
    const int lane = threadIdx.x & 31;
    const int64_t rows = (int64_t)g.lnz * g.ny, nch = (g.nx + 15) / 16;
    unsigned int bins[7] = {0, 0, 0, 0, 0, 0, 0};
    for (int64_t row = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; row < rows;
         row += ((int64_t)gridDim.x * blockDim.x) >> 5) {
        const int64_t y = row % g.ny, zl = row / g.ny;
        uint8_t *k = K + pidx(g, zl + 1, y, 0);
        for (int64_t c = lane; c < nch; c += 32) {
            uint4 w = *(const uint4 *)(k + 16 * c);
            if ((w.x | w.y | w.z | w.w) == 0) continue;
#pragma unroll
            for (int i = 0; i < 4; i++) {
                const uint32_t wi = swar::w4(w, i);
#pragma unroll
                for (int b = 0; b < 7; b++) bins[b] += __popc(swar::zero(wi ^ (0x80808080u | (0x01010101u * b))));
            }
            w.x &= 0x7F7F7F7Fu;
            w.y &= 0x7F7F7F7Fu;
            w.z &= 0x7F7F7F7Fu;
            w.w &= 0x7F7F7F7Fu;
            *(uint4 *)(k + 16 * c) = w;
        }
    }
#pragma unroll
    for (int b = 0; b < 7; b++) {
        unsigned int v = bins[b];
#pragma unroll
        for (int o = 16; o; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
        if (lane == 0 && v) atomicAdd(&h[b], (unsigned long long)v);
    }
    __syncthreads();
    if (threadIdx.x < 7 && h[threadIdx.x]) atomicAdd(&hist[threadIdx.x], h[threadIdx.x]);
}

// ---- ordered compaction of selected voxels, one warp per row (ascending x):
// the row's selection is counted (pass 1), the counts are scanned on the
// device, and each warp writes its row's entries at its offset (pass 2).
// sel(w4, k, c) returns a 16-byte flag vector (0x80 per selected byte) of chunk c.
enum RowSel { kSelBoundary = 0, kSelShell = 1 };

// boundary nodes: 0 < K < 6
static __device__ __forceinline__ uint4 sel_boundary(const uint8_t *k, int64_t c, const Grid &)
{
    const uint4 w = *(const uint4 *)(k + 16 * c);
    return make_uint4(swar::bnd(w.x), swar::bnd(w.y), swar::bnd(w.z), swar::bnd(w.w));
}

// shell voxels (twostep.cu): inside, and itself or a face neighbour a boundary
// node (K < 6; ghost planes hold 0x80-flagged bytes, which are not < 6)
static __device__ __forceinline__ uint4 sel_shell(const uint8_t *k, int64_t c, const Grid &g)
{
    const uint8_t *p = k + 16 * c;
    const uint4 w = *(const uint4 *)p;
    if ((w.x | w.y | w.z | w.w) == 0) return make_uint4(0, 0, 0, 0);
    const uint4 ym = *(const uint4 *)(p - g.pitch), yp = *(const uint4 *)(p + g.pitch);
    const uint4 zm = *(const uint4 *)(p - g.plane), zp = *(const uint4 *)(p + g.plane);
    const uint32_t before = (uint32_t)p[-1] << 24, after = p[16];
    const uint32_t six = 0x06060606u;
    uint32_t r[4];
#pragma unroll
    for (int i = 0; i < 4; i++) {
        const uint32_t wi = swar::w4(w, i);
        const uint32_t prev = i == 0 ? before : swar::w4(w, i - 1);
        const uint32_t next = i == 3 ? after : swar::w4(w, i + 1);
        const uint32_t near = swar::lt(wi, six) | swar::lt(swar::xm(wi, prev), six) | swar::lt(swar::xp(wi, next), six) |
                              swar::lt(swar::w4(ym, i), six) | swar::lt(swar::w4(yp, i), six) |
                              swar::lt(swar::w4(zm, i), six) | swar::lt(swar::w4(zp, i), six);
        r[i] = near & ~swar::zero(wi) & 0x80808080u;
    }
    return make_uint4(r[0], r[1], r[2], r[3]);
}

template <int SEL>
static __device__ __forceinline__ uint4 row_sel(const uint8_t *k, int64_t c, const Grid &g)
{
    return SEL == kSelBoundary ? sel_boundary(k, c, g) : sel_shell(k, c, g);
}

template <int SEL>
__global__ void k_rows_count(Grid g, const uint8_t *__restrict__ K, int64_t *__restrict__ counts)
{
    const int lane = threadIdx.x & 31;
    const int64_t rows = (int64_t)g.lnz * g.ny, nch = (g.nx + 15) / 16;
    for (int64_t row = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; row < rows;
         row += ((int64_t)gridDim.x * blockDim.x) >> 5) {
        const int64_t y = row % g.ny, zl = row / g.ny;
        const uint8_t *k = K + pidx(g, zl + 1, y, 0);
        int n = 0;
        for (int64_t c = lane; c < nch; c += 32) {
            const uint4 f = row_sel<SEL>(k, c, g);
            n += __popc(f.x) + __popc(f.y) + __popc(f.z) + __popc(f.w);
        }
#pragma unroll
        for (int o = 16; o; o >>= 1) n += __shfl_xor_sync(0xffffffffu, n, o);
        if (lane == 0) counts[row] = n;
    }
}

// out(i, pos, x, k): entry i is the voxel at padded offset pos, row x, value k
template <int SEL, typename Out>
static __device__ __forceinline__ void rows_compact(const Grid &g, const uint8_t *__restrict__ K,
                                                    const int64_t *__restrict__ row_off, Out out)
{
    const int lane = threadIdx.x & 31;
    const int64_t rows = (int64_t)g.lnz * g.ny, nch = (g.nx + 15) / 16;
    for (int64_t row = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; row < rows;
         row += ((int64_t)gridDim.x * blockDim.x) >> 5) {
        const int64_t y = row % g.ny, zl = row / g.ny;
        const int64_t base = pidx(g, zl + 1, y, 0);
        const uint8_t *k = K + base;
        int64_t o = row_off[row];
        if (row_off[row + 1] == o) continue;  // nothing selected in this row
        for (int64_t c0 = 0; c0 < nch; c0 += 32) {
            const int64_t c = c0 + lane;
            uint4 f = c < nch ? row_sel<SEL>(k, c, g) : make_uint4(0, 0, 0, 0);
            const int n = __popc(f.x) + __popc(f.y) + __popc(f.z) + __popc(f.w);
            int incl = n;
#pragma unroll
            for (int d = 1; d < 32; d <<= 1) {
                const int t = __shfl_up_sync(0xffffffffu, incl, d);
                if (lane >= d) incl += t;
            }
            int64_t at = o + incl - n;
#pragma unroll
            for (int i = 0; i < 4; i++) {
                uint32_t m = swar::w4(f, i);
                while (m) {
                    const int b = (__ffs(m) - 1) >> 3;  // byte index of the lowest selected byte
                    m &= m - 1;
                    const int64_t x = 16 * c + 4 * i + b;
                    out(at++, base + x, x, k[x]);
                }
            }
            o += __shfl_sync(0xffffffffu, incl, 31);
        }
    }
}

template <typename IdxT>
__global__ void k_compact(Grid g, const uint8_t *__restrict__ K, const int64_t *__restrict__ row_off,
                          int64_t zglob0, int32_t ny_glob, int32_t nx_glob, IdxT *__restrict__ bpos,
                          int64_t *__restrict__ bidx, uint8_t *__restrict__ Kb)
{
    rows_compact<kSelBoundary>(g, K, row_off, [&](int64_t i, int64_t pos, int64_t x, uint8_t kv) {
        const int64_t zl = pos / g.plane - 1, y = (pos % g.plane) / g.pitch - 1;
        bpos[i] = (IdxT)pos;
        bidx[i] = ((zglob0 + zl) * ny_glob + y) * nx_glob + x;
        Kb[i] = kv;
    });
}

// the shell list and, per entry, which of its six face neighbours are inside
// (bit 0..5: x-1, x+1, y-1, y+1, z-1, z+1; ghost-plane bytes carry the 0x80
// inside flag): the shell kernel loads only inside neighbours -- an outside
// voxel holds +0 -- and takes K as the popcount, so it reads no K byte
template <typename IdxT>
__global__ void k_shell_compact(Grid g, const uint8_t *__restrict__ K, const int64_t *__restrict__ off,
                                IdxT *__restrict__ list, uint8_t *__restrict__ nmask)
{
    rows_compact<kSelShell>(g, K, off, [&](int64_t i, int64_t pos, int64_t, uint8_t) {
        list[i] = (IdxT)pos;
        const int64_t d[6] = {-1, 1, -g.pitch, g.pitch, -g.plane, g.plane};
        uint32_t m = 0;
#pragma unroll
        for (int k = 0; k < 6; k++) m |= (K[pos + d[k]] != 0) << k;
        nmask[i] = (uint8_t)m;
    });
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

// one warp per row: blocks of 8 warps, at most 148 * 16 blocks (grid-stride)
static unsigned row_blocks(int64_t rows) { return grid_for(rows * 32, 256); }

cudaError_t launch_scatter_mask(const Grid &g, const uint8_t *mask_chunk, int zp0, int nzc,
                                uint8_t *K, cudaStream_t s)
{
    const int64_t rows = (int64_t)nzc * g.ny;
    if (rows == 0) return cudaSuccess;
    k_scatter_mask<<<row_blocks(rows), 256, 0, s>>>(g, mask_chunk, zp0, nzc, K);
    return cudaGetLastError();
}

// Bit-packed chunk (maskpack.cu): nzc planes from local padded plane zp0, rows
// of rw 32-bit words, bit i of word w = voxel x = 32 w + i.  One thread per
// word writes the 32 K bytes it covers (0x80 where set, as k_scatter_mask).
__global__ void k_scatter_mask_bits(Grid g, const uint32_t *__restrict__ bits, int rw, int zp0, int nzc,
                                    uint8_t *__restrict__ K)
{
    const int64_t nw = (int64_t)nzc * g.ny * rw;
    for (int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; t < nw; t += (int64_t)gridDim.x * blockDim.x) {
        const int64_t row = t / rw;
        const int wi = (int)(t - row * rw), x0 = 32 * wi;
        const int64_t y = row % g.ny, z = row / g.ny;
        const uint32_t b = bits[t];
        uint8_t *k = K + pidx(g, zp0 + z, y, x0);
        if (x0 + 32 <= g.nx) {  // x = 0 of a K row is 16-byte aligned, x0 a multiple of 32
            uint32_t e[8];
#pragma unroll
            for (int j = 0; j < 8; j++) e[j] = ((((b >> (4 * j)) & 15u) * 0x00204081u) & 0x01010101u) * 0x80u;
            *(uint4 *)k = make_uint4(e[0], e[1], e[2], e[3]);
            *(uint4 *)(k + 16) = make_uint4(e[4], e[5], e[6], e[7]);
        } else {
            for (int i = 0; i < g.nx - x0; i++) k[i] = ((b >> i) & 1u) ? 0x80 : 0;
        }
    }
}

cudaError_t launch_scatter_mask_bits(const Grid &g, const uint32_t *bits, int rw, int zp0, int nzc, uint8_t *K,
                                     cudaStream_t s)
{
    const int64_t nw = (int64_t)nzc * g.ny * rw;
    if (nw == 0) return cudaSuccess;
    k_scatter_mask_bits<<<grid_for(nw, 256), 256, 0, s>>>(g, bits, rw, zp0, nzc, K);
    return cudaGetLastError();
}

cudaError_t launch_count_k(const Grid &g, uint8_t *K, cudaStream_t s)
{
    const int64_t items = (int64_t)g.lnz * g.ny * ((g.nx + 15) / 16);
    if (items == 0) return cudaSuccess;
    k_count_k<<<grid_for(items), 256, 0, s>>>(g, K);
    return cudaGetLastError();
}

cudaError_t launch_finish_k(const Grid &g, uint8_t *K, unsigned long long *hist8, cudaStream_t s)
{
    const int64_t rows = (int64_t)g.lnz * g.ny;
    if (rows == 0) return cudaSuccess;
    k_finish_k<<<row_blocks(rows), 256, 0, s>>>(g, K, hist8);
    // the two ghost planes keep their 0x80 inside flags: set_state / read use
    // them to keep ghost values, the energy hook for cross-slab edges; no
    // kernel of the step reads K there
    return cudaGetLastError();
}

cudaError_t launch_row_counts64(const Grid &g, const uint8_t *K, int64_t *counts, cudaStream_t s)
{
    const int64_t rows = (int64_t)g.lnz * g.ny;
    if (rows == 0) return cudaSuccess;
    k_rows_count<kSelBoundary><<<row_blocks(rows), 256, 0, s>>>(g, K, counts);
    return cudaGetLastError();
}

cudaError_t launch_compact(const Grid &g, const uint8_t *K, const int64_t *row_off, int64_t zglob0,
                           int32_t ny_glob, int32_t nx_glob, bool idx64, void *bpos,
                           int64_t *bidx, uint8_t *Kb, cudaStream_t s)
{
    const int64_t rows = (int64_t)g.lnz * g.ny;
    if (rows == 0) return cudaSuccess;
    if (idx64)
        k_compact<int64_t><<<row_blocks(rows), 256, 0, s>>>(g, K, row_off, zglob0, ny_glob, nx_glob,
                                                             (int64_t *)bpos, bidx, Kb);
    else
        k_compact<uint32_t><<<row_blocks(rows), 256, 0, s>>>(g, K, row_off, zglob0, ny_glob, nx_glob,
                                                              (uint32_t *)bpos, bidx, Kb);
    return cudaGetLastError();
}

cudaError_t launch_shell_counts(const Grid &g, const uint8_t *K, int64_t *counts, cudaStream_t s)
{
    const int64_t rows = (int64_t)g.lnz * g.ny;
    if (rows == 0) return cudaSuccess;
    k_rows_count<kSelShell><<<row_blocks(rows), 256, 0, s>>>(g, K, counts);
    return cudaGetLastError();
}

cudaError_t launch_shell_compact(const Grid &g, const uint8_t *K, const int64_t *off, bool idx64, void *list,
                                 uint8_t *nmask, cudaStream_t s)
{
    const int64_t rows = (int64_t)g.lnz * g.ny;
    if (rows == 0) return cudaSuccess;
    if (idx64) k_shell_compact<int64_t><<<row_blocks(rows), 256, 0, s>>>(g, K, off, (int64_t *)list, nmask);
    else k_shell_compact<uint32_t><<<row_blocks(rows), 256, 0, s>>>(g, K, off, (uint32_t *)list, nmask);
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
