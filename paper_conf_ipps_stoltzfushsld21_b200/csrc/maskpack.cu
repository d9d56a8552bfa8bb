// maskpack.cu -- host side of the bit-packed mask upload (rafd_create from a
// host mask).  The voxel mask is one byte per voxel (include/rafd.h); moving
// it over PCIe costs 1 byte per voxel (C4: 1.1 GB, 20 ms at the link's 54
// GB/s), while the classification needs one bit.  Host threads pack each row
// into 32-bit words (bit i of word w = mask[32 w + i] != 0, the tail bits 0)
// into a pinned staging buffer, chunk by chunk, while the previous chunk is
// copied and expanded on the device (classify.cu, k_scatter_mask_bits).
#include <immintrin.h>
#include <stdint.h>
#include <string.h>

#include <algorithm>
#include <thread>
#include <vector>

namespace rafd {

// one row of nx mask bytes -> rw words
static void pack_row_scalar(const uint8_t *m, int nx, uint32_t *out, int rw)
{
    for (int w = 0; w < rw; w++) {
        uint32_t b = 0;
        const int x0 = 32 * w, n = std::min(32, nx - x0);
        for (int i = 0; i < n; i++) b |= (uint32_t)(m[x0 + i] != 0) << i;
        out[w] = b;
    }
}

__attribute__((target("avx2"))) static void pack_row_avx2(const uint8_t *m, int nx, uint32_t *out, int rw)
{
    const __m256i zero = _mm256_setzero_si256();
    const int full = nx / 32;
    for (int w = 0; w < full; w++) {
        const __m256i v = _mm256_loadu_si256((const __m256i *)(m + 32 * w));
        out[w] = ~(uint32_t)_mm256_movemask_epi8(_mm256_cmpeq_epi8(v, zero));
    }
    if (full < rw) {
        uint32_t b = 0;
        for (int i = 0; i < nx - 32 * full; i++) b |= (uint32_t)(m[32 * full + i] != 0) << i;
        out[full] = b;
    }
}

static bool have_avx2()
{
    static int v = -1;
    if (v < 0) v = __builtin_cpu_supports("avx2") ? 1 : 0;
    return v == 1;
}

int pack_threads()
{
    const unsigned h = std::thread::hardware_concurrency();
    return (int)std::max(1u, std::min(h ? h : 1u, 32u));
}

// rows [0, nrows) of nx bytes each (row stride nx) -> rows of rw words
void pack_mask_rows(const uint8_t *mask, int64_t nrows, int nx, uint32_t *out, int rw, int nthreads)
{
    const bool avx2 = have_avx2();
    auto work = [&](int64_t r0, int64_t r1) {
        for (int64_t r = r0; r < r1; r++) {
            if (avx2)
                pack_row_avx2(mask + r * nx, nx, out + r * rw, rw);
            else
                pack_row_scalar(mask + r * nx, nx, out + r * rw, rw);
        }
    };
    const int64_t per = (nrows + nthreads - 1) / nthreads;
    if (nthreads <= 1 || nrows < 64) {
        work(0, nrows);
        return;
    }
    std::vector<std::thread> th;
    th.reserve(nthreads);
    for (int t = 0; t < nthreads; t++) {
        const int64_t r0 = t * per, r1 = std::min(nrows, r0 + per);
        if (r0 >= r1) break;
        th.emplace_back(work, r0, r1);
    }
    for (auto &t : th) t.join();
}

}  // namespace rafd
