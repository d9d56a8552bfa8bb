// aux.cu -- off-hot-path kernels: state in/out (canonical <-> padded layout),
// the ub_prev refresh after set_state, and the discrete-energy test hook.
#include "internal.cuh"

namespace rafd {

static unsigned grid_for(int64_t n)
{
    int64_t b = (n + 255) / 256;
    if (b > 148 * 32) b = 148 * 32;
    return (unsigned)(b < 1 ? 1 : b);
}

// src_chunk holds nzc planes of the room starting at local padded plane zp0;
// values at K = 0 are stored as +0 (reading R15).
template <typename T>
__global__ void k_field_in(Grid g, const T *__restrict__ src, int zp0, int nzc,
                           const uint8_t *__restrict__ K, T *__restrict__ dst)
{
    const int64_t n = (int64_t)nzc * g.ny * g.nx;
    for (int64_t c = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; c < n;
         c += (int64_t)gridDim.x * blockDim.x) {
        const int64_t x = c % g.nx, r = c / g.nx, y = r % g.ny, z = r / g.ny;
        const int64_t p = (zp0 + z) * g.plane + (y + 1) * g.pitch + g.xo + x;
        dst[p] = K[p] ? src[c] : (T)0;
    }
}

template <typename T>
__global__ void k_field_out(Grid g, const T *__restrict__ src, int zp0, int nzc, T *__restrict__ dst)
{
    const int64_t n = (int64_t)nzc * g.ny * g.nx;
    for (int64_t c = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; c < n;
         c += (int64_t)gridDim.x * blockDim.x) {
        const int64_t x = c % g.nx, r = c / g.nx, y = r % g.ny, z = r / g.ny;
        dst[c] = src[(zp0 + z) * g.plane + (y + 1) * g.pitch + g.xo + x];
    }
}

template <typename T, typename IdxT>
__global__ void k_gather_ub(const IdxT *__restrict__ bpos, int64_t Nb, const T *__restrict__ u,
                            T *__restrict__ ub)
{
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < Nb;
         i += (int64_t)gridDim.x * blockDim.x)
        ub[i] = u[(int64_t)bpos[i]];
}

template <typename T>
cudaError_t launch_field_in(const Grid &g, const T *src_chunk, int zp0, int nzc, const uint8_t *K,
                            T *dst, cudaStream_t s)
{
    const int64_t n = (int64_t)nzc * g.ny * g.nx;
    if (n == 0) return cudaSuccess;
    k_field_in<T><<<grid_for(n), 256, 0, s>>>(g, src_chunk, zp0, nzc, K, dst);
    return cudaGetLastError();
}

template <typename T>
cudaError_t launch_field_out(const Grid &g, const T *src, int zp0, int nzc, T *dst_chunk,
                             cudaStream_t s)
{
    const int64_t n = (int64_t)nzc * g.ny * g.nx;
    if (n == 0) return cudaSuccess;
    k_field_out<T><<<grid_for(n), 256, 0, s>>>(g, src, zp0, nzc, dst_chunk);
    return cudaGetLastError();
}

template <typename T>
cudaError_t launch_gather_ub(const void *bpos, bool idx64, int64_t Nb, const T *u, T *ub,
                             cudaStream_t s)
{
    if (Nb == 0) return cudaSuccess;
    if (idx64) k_gather_ub<T, int64_t><<<grid_for(Nb), 256, 0, s>>>((const int64_t *)bpos, Nb, u, ub);
    else k_gather_ub<T, uint32_t><<<grid_for(Nb), 256, 0, s>>>((const uint32_t *)bpos, Nb, u, ub);
    return cudaGetLastError();
}

// ---------------------------------------------------------------- energy
// H^{n+1/2} (reading R11) = kin + l^2 pot + bnd, accumulated in double:
//   kin = sum over inside voxels of (u^{n+1} - u^n)^2
//   pot = sum over inside edges (i,j) of (u^{n+1}_i - u^{n+1}_j)(u^n_i - u^n_j)
//         (edges to +x, +y, +z; +z may reach the upper ghost plane of a slab,
//          whose K holds the inside flag)
//   bnd = sum over boundary nodes of l (6-K) sum_b (D v^2 + F g^2)
static __device__ __forceinline__ double warp_sum(double v)
{
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    return v;
}

template <typename T>
__global__ void k_energy_vol(Grid g, const T *__restrict__ un1, const T *__restrict__ un,
                             const uint8_t *__restrict__ K, double *acc)
{
    double kin = 0, pot = 0;
    const int64_t n = (int64_t)g.lnz * g.ny * g.nx;
    for (int64_t c = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; c < n;
         c += (int64_t)gridDim.x * blockDim.x) {
        const int64_t x = c % g.nx, r = c / g.nx, y = r % g.ny, z = r / g.ny;
        const int64_t i = (z + 1) * g.plane + (y + 1) * g.pitch + g.xo + x;
        if (K[i] == 0) continue;
        const double a1 = (double)un1[i], a0 = (double)un[i];
        kin += (a1 - a0) * (a1 - a0);
        const int64_t nb[3] = {i + 1, i + g.pitch, i + g.plane};
#pragma unroll
        for (int k = 0; k < 3; k++) {
            const int64_t j = nb[k];
            if (K[j] == 0) continue;
            pot += (a1 - (double)un1[j]) * (a0 - (double)un[j]);
        }
    }
    kin = warp_sum(kin);
    pot = warp_sum(pot);
    if ((threadIdx.x & 31) == 0) {
        atomicAdd(&acc[0], kin);
        atomicAdd(&acc[1], pot);
    }
}

template <typename T>
__global__ void k_energy_bnd(const uint8_t *__restrict__ Kb, const uint8_t *__restrict__ matb,
                             int64_t Nb, int MB, const T *__restrict__ v, const T *__restrict__ gs,
                             const double *__restrict__ DF, int M, double lambda, double *acc)
{
    double e = 0;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < Nb;
         i += (int64_t)gridDim.x * blockDim.x) {
        const int m = matb[i];
        double s = 0;
        for (int b = 0; b < MB; b++) {
            const double vb = (double)v[(int64_t)b * Nb + i], gb = (double)gs[(int64_t)b * Nb + i];
            s += DF[m * MB + b] * vb * vb + DF[M * MB + m * MB + b] * gb * gb;
        }
        e += lambda * (double)(6 - Kb[i]) * s;
    }
    e = warp_sum(e);
    if ((threadIdx.x & 31) == 0) atomicAdd(&acc[2], e);
}

template <typename T>
cudaError_t launch_energy(const Grid &g, const T *un1, const T *un, const uint8_t *K, double *acc,
                          cudaStream_t s)
{
    const int64_t n = (int64_t)g.lnz * g.ny * g.nx;
    k_energy_vol<T><<<grid_for(n), 256, 0, s>>>(g, un1, un, K, acc);
    return cudaGetLastError();
}

template <typename T>
cudaError_t launch_energy_bnd(const uint8_t *Kb, const uint8_t *matb, int64_t Nb, int MB,
                              const T *v, const T *gst, const double *DF, int M, double lambda,
                              double *acc, cudaStream_t s)
{
    if (MB == 0 || Nb == 0) return cudaSuccess;
    k_energy_bnd<T><<<grid_for(Nb), 256, 0, s>>>(Kb, matb, Nb, MB, v, gst, DF, M, lambda, acc);
    return cudaGetLastError();
}

#define RAFD_INST(T)                                                                              \
    template cudaError_t launch_field_in<T>(const Grid &, const T *, int, int, const uint8_t *,   \
                                            T *, cudaStream_t);                                   \
    template cudaError_t launch_field_out<T>(const Grid &, const T *, int, int, T *, cudaStream_t); \
    template cudaError_t launch_gather_ub<T>(const void *, bool, int64_t, const T *, T *,         \
                                             cudaStream_t);                                       \
    template cudaError_t launch_energy<T>(const Grid &, const T *, const T *, const uint8_t *,    \
                                          double *, cudaStream_t);                                \
    template cudaError_t launch_energy_bnd<T>(const uint8_t *, const uint8_t *, int64_t, int,     \
                                              const T *, const T *, const double *, int, double,  \
                                              double *, cudaStream_t);
RAFD_INST(float)
RAFD_INST(double)
#undef RAFD_INST
template cudaError_t launch_field_out<uint8_t>(const Grid &, const uint8_t *, int, int, uint8_t *,
                                                cudaStream_t);

}  // namespace rafd
