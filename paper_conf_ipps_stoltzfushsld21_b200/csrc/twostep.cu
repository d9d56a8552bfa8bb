// twostep.cu -- temporal blocking: two leapfrog steps per HBM sweep (SURVEY
// §8(f) row f4).
//
// The volume update (Listing 2 kernel 1) of step n+1 at a
// voxel needs u^n on its 7-point star; that of step n+2 needs u^{n+1} there.
// One z-march can therefore produce both levels: the CTA computes u^{n+1} of
// plane q (kept in shared memory and registers) and, one plane behind, u^{n+2}
// of plane q-1 from it.  Per voxel and double step it reads u^{n-1}, u^n, K and
// writes u^{n+1}, u^{n+2}: 4s+1 bytes for two steps instead of 2(3s+1).
//
// Three things make this exact (bitwise equal to two single steps):
//  * out of place: u^{n-1}, u^n are read from one buffer pair and u^{n+1},
//    u^{n+2} written to the other (four field buffers), so overlapping tiles
//    never read a value another CTA has already advanced;
//  * overlapped tiles: the u^{n+1} a tile's step n+2 needs from its x/y
//    neighbours is recomputed (step n+1 runs on the tile plus one ring of
//    voxels; 30 of the 32 lane vectors, TY of the TY+2 rows are stored);
//  * the "shell": a voxel's u^{n+2} from this kernel is final only if neither
//    the voxel nor a face neighbour is a boundary node (their u^{n+1} changes
//    in the boundary kernel, rows a3/a4) or the source voxel (row a5).  Those
//    voxels (a list built once per room; the source and its neighbours in a
//    7-entry side list) are recomputed by k_shell after the boundary kernel
//    and the source injection of step n+1, with the same arithmetic.
//
// Sequence of one double step (room.cu, enqueue_step2):
//   k_volume2 (A=u^{n-1}, B=u^n -> C=u^{n+1}, D=u^{n+2} provisional)
//   k_boundary(C), k_src_rcv(C)          -- step n+1 final
//   k_shell   (C, B -> D at shell voxels) -- step n+2 volume final
//   k_boundary(D), k_src_rcv(D)          -- step n+2 final
#include <cuda.h>
#include <cudaTypedefs.h>

#include <stdlib.h>

#include "bnd_math.cuh"
#include "internal.cuh"

namespace rafd {

// ------------------------------------------------------------------ PTX helpers
namespace tb {
static __device__ __forceinline__ uint32_t smem_u32(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }
static __device__ __forceinline__ void mbar_init(uint64_t *b, uint32_t count)
{
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(b)), "r"(count));
}
static __device__ __forceinline__ void mbar_expect_tx(uint64_t *b, uint32_t bytes)
{
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(b)), "r"(bytes) : "memory");
}
static __device__ __forceinline__ void mbar_wait(uint64_t *b, uint32_t parity)
{
    asm volatile(
        "{\n\t.reg .pred p;\n"
        "WAIT_%=:\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
        "@!p bra WAIT_%=;\n\t}" ::"r"(smem_u32(b)),
        "r"(parity)
        : "memory");
}
static __device__ __forceinline__ void tma_load_3d(void *dst, const CUtensorMap *map, uint64_t *bar, int c0, int c1,
                                                   int c2)
{
    asm volatile(
        "cp.async.bulk.tensor.3d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, "
        "%4}], [%5];" ::"r"(smem_u32(dst)),
        "l"((uint64_t)map), "r"(c0), "r"(c1), "r"(c2), "r"(smem_u32(bar))
        : "memory");
}
static __device__ __forceinline__ uint64_t policy_evict_first()
{
    uint64_t p;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
    return p;
}
static __device__ __forceinline__ void st_v4_hint(void *ptr, uint4 v, uint64_t pol)
{
    asm volatile("st.global.L2::cache_hint.v4.b32 [%0], {%1, %2, %3, %4}, %5;" ::"l"(ptr), "r"(v.x), "r"(v.y),
                 "r"(v.z), "r"(v.w), "l"(pol)
                 : "memory");
}
}  // namespace tb

template <typename T> struct Vec16;
template <> struct Vec16<float> {
    static constexpr int N = 4;
    using K = uint32_t;
};
template <> struct Vec16<double> {
    static constexpr int N = 2;
    using K = uint16_t;
};

// Tile geometry.  Step n+1 runs on TX x (TY+2) voxels (32 lanes x one 16-byte
// vector, rows -1..TY), step n+2 and both stores on the TXO x TY core (lanes
// 1..30, rows 0..TY-1); u^n is staged with one more ring (a vector in x, a
// row in y).  SU u^n slots, SP u^{n-1}/K slots, two u^{n+1} planes.
template <typename T, int TY, int SU, int SP> struct TbGeom {
    static constexpr int VEC = Vec16<T>::N;
    static constexpr int TX = 32 * VEC;
    static constexpr int TXO = TX - 2 * VEC;
    static constexpr int UROW = TX + 2 * VEC;
    static constexpr int UR = TY + 4, PR = TY + 2;
    static constexpr int NW = PR / 2;  // two step-(n+1) rows per warp
    static constexpr int NT = 32 * NW;
    static constexpr int U_BYTES = (UR * UROW * (int)sizeof(T) + 127) / 128 * 128;
    static constexpr int P_BYTES = PR * TX * (int)sizeof(T);
    // the K box starts at the 16-byte aligned byte at or below the region (TMA
    // box origins must be 16-byte aligned) and is 16 bytes wider
    static constexpr int KROW = TX + 16;
    static constexpr int K_BYTES = (PR * KROW + 127) / 128 * 128;
    static constexpr int U1_BYTES = PR * TX * (int)sizeof(T);
    static constexpr int U_TX = UR * UROW * (int)sizeof(T);
    static constexpr int PK_TX = P_BYTES + PR * KROW;
    static constexpr int SMEM = SU * U_BYTES + SP * (P_BYTES + K_BYTES) + 2 * U1_BYTES + (SU + SP) * 8 + 128;
    static_assert(PR % 2 == 0, "TY must be even");
};

// (T)K of byte i of a K word, exactly, without the XU conversion unit: the
// byte placed in the mantissa of 2^23 (2^52), minus 2^23 (2^52).  Measured:
// 3.47 -> 3.40 ms per C4 double step against I2F.U8.
template <typename T> static __device__ __forceinline__ T k_as(uint32_t kw, int i);
template <> __device__ __forceinline__ float k_as<float>(uint32_t kw, int i)
{
    return __fsub_rn(__int_as_float((int)__byte_perm(kw, 0x4Bu, 0x4550u | (uint32_t)i)), 8388608.0f);
}
template <> __device__ __forceinline__ double k_as<double>(uint32_t kw, int i)
{
    return __dsub_rn(__hiloint2double(0x43300000, (int)((kw >> (8 * i)) & 0xffu)), 4503599627370496.0);
}

// One 16-byte vector of the volume update (DESIGN.md §4 order): neighbours
// summed x-1, x+1, y-1, y+1, z-1, z+1; K = 0 keeps `keep` (outside: +0).
template <typename T>
static __device__ __forceinline__ void vol_vec(const T *c, const T *ym, const T *yp, const T *zm, const T *zp,
                                               const T *pv, T left, T right, uint32_t kw, T l2, T *o)
{
    using R = rn<T>;
    constexpr int VEC = Vec16<T>::N;
#pragma unroll
    for (int i = 0; i < VEC; i++) {
        const T kf = k_as<T>(kw, i);
        const T xm = i == 0 ? left : c[i - 1];
        const T xp = i == VEC - 1 ? right : c[i + 1];
        T s = R::add(xm, xp);
        s = R::add(s, ym[i]);
        s = R::add(s, yp[i]);
        s = R::add(s, zm[i]);
        s = R::add(s, zp[i]);
        const T a = R::sub((T)2, R::mul(l2, kf));
        T t = R::mul(a, c[i]);
        t = R::add(t, R::mul(l2, s));
        o[i] = kf != (T)0 ? R::sub(t, pv[i]) : pv[i];
    }
}

// The two-step kernel.  umap: u^n (box UROW x (TY+4)); pmap: u^{n-1} (TX x
// (TY+2)); kmap: K (TX x (TY+2)); out1 = u^{n+1}, out2 = u^{n+2} (other pair).
template <typename T, int TY, int SU, int SP, bool DYN>
__global__ void __launch_bounds__(TbGeom<T, TY, SU, SP>::NT, 1)
    k_volume2(const __grid_constant__ CUtensorMap umap, const __grid_constant__ CUtensorMap pmap,
              const __grid_constant__ CUtensorMap kmap, T *__restrict__ out1, T *__restrict__ out2, Grid g, T l2,
              int z_lo, int z_hi, int zchunk, int tiles_x, int tiles_y, unsigned int *work)
{
    using G = TbGeom<T, TY, SU, SP>;
    using KW = typename Vec16<T>::K;
    constexpr int VEC = G::VEC, TX = G::TX, TXO = G::TXO, UROW = G::UROW;
    // The dynamic shared window starts 1 KB-aligned (checked below): every slot
    // is the array plus a compile-time offset (LDS/STS, no runtime alignment).
    extern __shared__ __align__(1024) unsigned char smem_raw[];
    unsigned char *const base = smem_raw;
    T *us = (T *)base;                                                  // SU u^n slots
    T *ps = (T *)(base + SU * G::U_BYTES);                              // SP u^{n-1} slots
    uint8_t *ks = base + SU * G::U_BYTES + SP * G::P_BYTES;             // SP K slots
    T *u1s = (T *)(base + SU * G::U_BYTES + SP * (G::P_BYTES + G::K_BYTES));  // 2 u^{n+1} planes
    uint64_t *bar = (uint64_t *)((unsigned char *)u1s + 2 * G::U1_BYTES);
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;

    static_assert((SU & (SU - 1)) == 0 && (SP & (SP - 1)) == 0, "ring sizes are powers of two");
    if (tid == 0) {
        if (tb::smem_u32(smem_raw) & 127u) __trap();  // TMA destinations need 128-byte alignment
        for (int i = 0; i < SU + SP; i++) tb::mbar_init(&bar[i], 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    uint32_t uph = 0, pph = 0;
    const uint64_t pol = tb::policy_evict_first();

    // stored planes: local [z_lo, z_hi) (a z slab stores its interior planes;
    // the u^n ghost planes it reads are the neighbours' edge planes)
    const int nz = z_hi - z_lo;
    const int nchunks = (nz + zchunk - 1) / zchunk;
    const int tiles = tiles_x * tiles_y;
    const int units = nchunks * tiles;
    // this warp's two step-(n+1) rows, relative to the tile's first core row
    const int r0 = 2 * warp - 1;
    // Units in (chunk, tile-y, tile-x) order, handed out dynamically (work != null:
    // an atomic counter, reset by the last CTA) so the units in flight stay the
    // next ~gridDim.x ones and neighbouring tiles march their planes together; or
    // statically round-robin.  Each CTA reserves its next unit when it starts one.
    int *const s_next = (int *)(bar + SU + SP);
    int unit = blockIdx.x, next_unit = 0;
    if constexpr (DYN) {
        if (tid == 0) *s_next = (int)atomicAdd(work, 1u);
        __syncthreads();
        unit = *s_next;
    }
    while (unit < units) {
        if constexpr (DYN) {
            if (tid == 0) next_unit = (int)atomicAdd(work, 1u);
        }
        const int chunk = unit / tiles, t = unit % tiles;
        const int ty = t / tiles_x, tx = t % tiles_x;
        const int pa = 1 + z_lo + chunk * zchunk;   // first padded plane stored
        const int pb = min(1 + z_hi, pa + zchunk);  // one past the last
        const int ox = tx * TXO, oy = ty * TY;      // core origin (room coordinates)
        const int ux = g.xo + ox - 2 * VEC;         // u^n box origin (padded x)
        const int uy = oy - 1;                      // padded row of core row -2
        const int px = g.xo + ox - VEC, py = oy;    // u^{n-1} box origin (padded)
        const int kx = px + k_shift(g);              // K bytes of the region start
        const int kd = kx & 15;                      // its offset in the aligned K box
        auto issue_u = [&](int p) {
            const int s = (p + 2) & (SU - 1);
            tb::mbar_expect_tx(&bar[s], G::U_TX);
            tb::tma_load_3d((unsigned char *)us + s * G::U_BYTES, &umap, &bar[s], ux, uy, p);
        };
        auto issue_pk = [&](int p) {
            const int s = (p + 1) & (SP - 1);
            tb::mbar_expect_tx(&bar[SU + s], G::PK_TX);
            tb::tma_load_3d((unsigned char *)ps + s * G::P_BYTES, &pmap, &bar[SU + s], px, py, p);
            tb::tma_load_3d(ks + s * G::K_BYTES, &kmap, &bar[SU + s], kx - kd, py, p);
        };
        auto wait_u = [&](int p) {
            const int s = (p + 2) & (SU - 1);
            tb::mbar_wait(&bar[s], (uph >> s) & 1);
            uph ^= 1u << s;
        };
        auto wait_pk = [&](int p) {
            const int s = (p + 1) & (SP - 1);
            tb::mbar_wait(&bar[SU + s], (pph >> s) & 1);
            pph ^= 1u << s;
        };
        auto uslot = [&](int p) -> const T * { return us + ((p + 2) & (SU - 1)) * (G::U_BYTES / (int)sizeof(T)); };
        // u^n planes pa-2 .. pb+1, u^{n-1}/K planes pa-1 .. pb
        __syncthreads();  // the previous unit is done with every slot
        if (tid == 0) {
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
            for (int p = pa - 2; p < pa - 2 + SU && p <= pb + 1; p++) issue_u(p);
            for (int p = pa - 1; p < pa - 1 + SP && p <= pb; p++) issue_pk(p);
        }
        // register windows per row k: u^n at q-1 and q, u^{n+1} at q-2 and q-1, K at q-1
        T unm[2][VEC], unc[2][VEC], o1m[2][VEC], o1c[2][VEC];
        KW km[2];
        wait_u(pa - 2);
        wait_u(pa - 1);
        const int col = VEC + lane * VEC;  // this lane's vector in a u^n smem row
#pragma unroll
        for (int k = 0; k < 2; k++) {
            const int sr = r0 + k + 2;  // smem row of step row r in the u^n box
            *(uint4 *)unm[k] = *(const uint4 *)(uslot(pa - 2) + sr * UROW + col);
            *(uint4 *)unc[k] = *(const uint4 *)(uslot(pa - 1) + sr * UROW + col);
#pragma unroll
            for (int i = 0; i < VEC; i++) o1m[k][i] = o1c[k][i] = (T)0;
            km[k] = 0;
        }
        __syncthreads();  // plane pa-2 lives on in registers only: refill its slot
        if (tid == 0) {
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
            if (pa - 2 + SU <= pb + 1) issue_u(pa - 2 + SU);
        }
        const bool lane_core = lane >= 1 && lane <= 30;
        const int xv = ox + (lane - 1) * VEC;        // room x of this lane's vector (core lanes)
        const bool x_ok = lane_core && xv < g.nx;
        for (int q = pa - 1; q <= pb; q++) {
            wait_u(q + 1);
            wait_pk(q);
            const T *uq = uslot(q), *uqp = uslot(q + 1);
            const T *pq = ps + ((q + 1) & (SP - 1)) * (G::P_BYTES / (int)sizeof(T));
            const uint8_t *kq = ks + ((q + 1) & (SP - 1)) * G::K_BYTES;
            T *u1w = u1s + (q & 1) * (G::U1_BYTES / (int)sizeof(T));
            T o1p[2][VEC], unp[2][VEC];
            KW kqv[2];
            // ---- step n+1 on plane q, rows r0, r0+1 (-1 .. TY)
#pragma unroll
            for (int k = 0; k < 2; k++) {
                const int r = r0 + k, sr = r + 2;
                T ym[VEC], yp[VEC], pv[VEC];
                *(uint4 *)unp[k] = *(const uint4 *)(uqp + sr * UROW + col);
                *(uint4 *)ym = *(const uint4 *)(uq + (sr - 1) * UROW + col);
                *(uint4 *)yp = *(const uint4 *)(uq + (sr + 1) * UROW + col);
                *(uint4 *)pv = *(const uint4 *)(pq + (r + 1) * TX + lane * VEC);
                kqv[k] = *(const KW *)(kq + (r + 1) * G::KROW + kd + lane * VEC);
                // the x halo of lanes 0 / 31 into registers of their own, loaded
                // before the shuffles (one load and one shuffle in flight together,
                // not a shuffle, then a load into the same register)
                T hl = (T)0, hr = (T)0;
                if (lane == 0) hl = uq[sr * UROW + VEC - 1];
                if (lane == 31) hr = uq[sr * UROW + VEC + TX];
                T left = __shfl_up_sync(0xffffffffu, unc[k][VEC - 1], 1);
                T right = __shfl_down_sync(0xffffffffu, unc[k][0], 1);
                left = lane == 0 ? hl : left;
                right = lane == 31 ? hr : right;
                vol_vec<T>(unc[k], ym, yp, unm[k], unp[k], pv, left, right, (uint32_t)kqv[k], l2, o1p[k]);
                *(uint4 *)(u1w + (r + 1) * TX + lane * VEC) = *(const uint4 *)o1p[k];
                if (q >= pa && q < pb && r >= 0 && r < TY && x_ok && oy + r < g.ny) {
                    T *dst = out1 + (int64_t)q * g.plane + (int64_t)(oy + r + 1) * g.pitch + g.xo + xv;
                    tb::st_v4_hint(dst, *(const uint4 *)o1p[k], pol);
                }
            }
            __syncthreads();  // u^{n+1} of plane q complete in shared memory
            // ---- step n+2 on plane q-1 (rows 0 .. TY-1, core lanes store)
            if (q - 1 >= pa) {
                const T *u1r = u1s + ((q - 1) & 1) * (G::U1_BYTES / (int)sizeof(T));
#pragma unroll
                for (int k = 0; k < 2; k++) {
                    // every warp runs both rows (uniform control flow, no divergent
                    // shuffles); the halo rows -1 and TY of warps 0 and NW-1 read a
                    // clamped row and are not stored
                    const int r = r0 + k, rr = min(max(r, 0), TY - 1);
                    T ym[VEC], yp[VEC], o2[VEC];
                    *(uint4 *)ym = *(const uint4 *)(u1r + rr * TX + lane * VEC);
                    *(uint4 *)yp = *(const uint4 *)(u1r + (rr + 2) * TX + lane * VEC);
                    const T left = __shfl_up_sync(0xffffffffu, o1c[k][VEC - 1], 1);
                    const T right = __shfl_down_sync(0xffffffffu, o1c[k][0], 1);
                    vol_vec<T>(o1c[k], ym, yp, o1m[k], o1p[k], unm[k], left, right, (uint32_t)km[k], l2, o2);
                    if (r >= 0 && r < TY && x_ok && oy + r < g.ny) {
                        T *dst = out2 + (int64_t)(q - 1) * g.plane + (int64_t)(oy + r + 1) * g.pitch + g.xo + xv;
                        tb::st_v4_hint(dst, *(const uint4 *)o2, pol);
                    }
                }
            }
#pragma unroll
            for (int k = 0; k < 2; k++) {
#pragma unroll
                for (int i = 0; i < VEC; i++) {
                    o1m[k][i] = o1c[k][i];
                    o1c[k][i] = o1p[k][i];
                    unm[k][i] = unc[k][i];
                    unc[k][i] = unp[k][i];
                }
                km[k] = kqv[k];
            }
            __syncthreads();  // u^n(q), u^{n-1}/K(q), u^{n+1}(q-1) no longer read
            if (tid == 0) {
                asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
                if (q + SU <= pb + 1) issue_u(q + SU);  // into the slot of plane q
                if (q + SP <= pb) issue_pk(q + SP);
            }
        }
        if constexpr (DYN) {
            if (tid == 0) *s_next = next_unit;
            __syncthreads();
            unit = *s_next;
        } else {
            unit += gridDim.x;
        }
    }
    if (DYN && tid == 0) {
        __threadfence();
        if (atomicAdd(work + 1, 1u) == gridDim.x - 1) {  // every CTA has taken its last unit
            atomicExch(work, 0u);
            atomicExch(work + 1, 0u);
        }
    }
}

// ------------------------------------------------------------------ the shell
// (the list -- inside voxels that are, or have a face neighbour that is, a
// boundary node -- is built by classify.cu's row compaction)

// u^{n+2} at the shell voxels and the source's 7-point star (src[7], -1 =
// none), from the final u^{n+1} (u1) and u^n (u0): the volume update in the
// order of DESIGN.md §4 (same expression as vol_vec).
// A slab recomputes only its interior planes (padded [zp_lo, zp_hi)): the list
// is then the sub-range of those planes and star entries elsewhere are skipped
// (its edge planes are recomputed whole from the exchanged u^{n+1}).
template <typename T, typename IdxT>
__global__ void __launch_bounds__(256) k_shell(const IdxT *__restrict__ list, const uint8_t *__restrict__ nmask,
                                               int64_t n, const int64_t *__restrict__ src,
                                               const T *__restrict__ u1, const T *__restrict__ u0,
                                               const uint8_t *__restrict__ K, T *__restrict__ out, Grid g, T l2,
                                               int zp_lo, int zp_hi)
{
    using R = rn<T>;
    const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= n + 7) return;
    const int64_t p = i < n ? (int64_t)list[i] : src[i - n];
    if (p < 0) return;
    if (i >= n && (p < (int64_t)zp_lo * g.plane || p >= (int64_t)zp_hi * g.plane)) return;
    // which face neighbours are inside: list entries carry it (no K load);
    // the source's star entries read K.  An outside neighbour holds +0, so it
    // is not loaded.  Every load depends only on p and the mask: all of them in
    // flight together.
    uint32_t m;
    int nbr;
    if (i < n) {
        m = nmask[i];
        nbr = __popc(m);
    } else {
        const int64_t d[6] = {-1, 1, -g.pitch, g.pitch, -g.plane, g.plane};
        m = 0;
#pragma unroll
        for (int k = 0; k < 6; k++) m |= (K[p + d[k]] != 0) << k;
        nbr = K[p];
    }
    const T xm = (m & 1) ? u1[p - 1] : (T)0, xp = (m & 2) ? u1[p + 1] : (T)0;
    const T ym = (m & 4) ? u1[p - g.pitch] : (T)0, yp = (m & 8) ? u1[p + g.pitch] : (T)0;
    const T zm = (m & 16) ? u1[p - g.plane] : (T)0, zp = (m & 32) ? u1[p + g.plane] : (T)0;
    const T c = u1[p], pv = u0[p];
    T s = R::add(xm, xp);
    s = R::add(s, ym);
    s = R::add(s, yp);
    s = R::add(s, zm);
    s = R::add(s, zp);
    const T a = R::sub((T)2, R::mul(l2, (T)nbr));
    T t = R::mul(a, c);
    t = R::add(t, R::mul(l2, s));
    // an outside voxel (a star entry with K = 0) holds +0 in every buffer, so
    // storing u0 there changes nothing
    out[p] = nbr != 0 ? R::sub(t, pv) : pv;
}

// ---- the shell fused with the step-(n+2) boundary update (whole rooms).
// Every boundary node is a shell voxel, and the shell list and the node list
// are both in ascending position order, so the k-th node entry of the shell
// list is node k: its index is the node count of the entry's 32-entry group
// (wbase, built with the plan) plus the nodes before it in its warp (ballot).
// Per entry: the volume value of step n+2 from the final u^{n+1} (as k_shell),
// then, at a node, Listing 3/4's update of it with the node's state (as
// k_boundary, DESIGN.md §4 order), one store of the final value.  The last
// block adds the source and records the receivers (as k_boundary).  The
// source's star entries that are shell voxels are left to their list entry.
// The list range [lo, hi) (a slab's interior phase: the sub-range of its
// interior planes, whose node entries are the interior nodes); threads start at
// the 32-entry group boundary below lo so every warp's ballot covers one whole
// group (entries below lo are counted, not processed).  Star entries are
// recomputed only inside the padded planes [zp_lo, zp_hi).  src_mode: as
// k_boundary's (3: add the source and record receivers; 2: record only).
template <typename T, int MB, typename IdxT, int ENT>
__global__ void __launch_bounds__(256)
    k_shell_bnd(const IdxT *__restrict__ list, const uint8_t *__restrict__ nmask, const int64_t *__restrict__ wbase,
                int64_t lo, int64_t hi, const int64_t *__restrict__ src, const T *__restrict__ u1,
                const T *__restrict__ u0, const uint8_t *__restrict__ K, T *__restrict__ out, Grid g, T l2, T l,
                const uint8_t *__restrict__ matb, T *__restrict__ ub, T *__restrict__ gst, T *__restrict__ vst,
                int64_t Nb, const T *__restrict__ tab, int M, Ctl<T> *ctl, unsigned int *ticket, int zp_lo,
                int zp_hi, int src_mode)
{
    using R = rn<T>;
    const int lane = threadIdx.x & 31;
    const int64_t lo32 = lo & ~(int64_t)31, nrange = hi - lo32;
    // ENT entries per thread (entry = block * 256 * ENT + e * 256 + tid): each
    // warp still covers 32 consecutive entries per e, and the block's ticket
    // below is paid once per 256 * ENT entries
#pragma unroll
    for (int e = 0; e < ENT; e++) {
        const int64_t j = (int64_t)blockIdx.x * (256 * ENT) + e * 256 + threadIdx.x;
        const int64_t i = lo32 + j;  // list index of a list thread
        const bool in_list = j < nrange;
        int64_t p = -1;
        uint32_t m = 0;
        int nbr = 0;
        if (in_list) {
            m = nmask[i];
            nbr = __popc(m);
            if (i >= lo) p = (int64_t)list[i];
        } else if (j < nrange + 7) {
            p = src[j - nrange];
            if (p >= 0 && (p < (int64_t)zp_lo * g.plane || p >= (int64_t)zp_hi * g.plane)) p = -1;
            if (p >= 0) {  // a star voxel: recomputed here unless it is a shell voxel (its list entry does it)
                const int64_t d[6] = {-1, 1, -g.pitch, g.pitch, -g.plane, g.plane};
                nbr = K[p];
                bool shell = nbr < 6;
#pragma unroll
                for (int k = 0; k < 6; k++) {
                    const int kn = K[p + d[k]];
                    m |= (kn != 0) << k;
                    shell = shell || kn < 6;
                }
                if (nbr == 0 || shell) p = -1;
            }
        }
        const bool node = in_list && nbr < 6;
        const unsigned bal = __ballot_sync(0xffffffffu, node);
        const int64_t rank = node ? wbase[i >> 5] + __popc(bal & ((1u << lane) - 1u)) : 0;
        if (p < 0) continue;  // below lo, or a star voxel left to its list entry
        if (p >= 0) {
            T uprev = (T)0, gb[MB > 0 ? MB : 1], vb[MB > 0 ? MB : 1];
            int mi = 0;
            if (node) {  // issued with the stencil loads
                mi = matb[rank];
                uprev = ub[rank];
#pragma unroll
                for (int b = 0; b < MB; b++) {
                    gb[b] = gst[(int64_t)b * Nb + rank];
                    vb[b] = vst[(int64_t)b * Nb + rank];
                }
            }
            const T xm = (m & 1) ? u1[p - 1] : (T)0, xp = (m & 2) ? u1[p + 1] : (T)0;
            const T ym = (m & 4) ? u1[p - g.pitch] : (T)0, yp = (m & 8) ? u1[p + g.pitch] : (T)0;
            const T zm = (m & 16) ? u1[p - g.plane] : (T)0, zp = (m & 32) ? u1[p + g.plane] : (T)0;
            // at a node u^n is its u_b slot (loaded above as uprev, the same value the
            // boundary update uses): the grid copy is read only at the other entries
            const T c = u1[p], pv = node ? uprev : u0[p];
            T s = R::add(xm, xp);
            s = R::add(s, ym);
            s = R::add(s, yp);
            s = R::add(s, zm);
            s = R::add(s, zp);
            const T a = R::sub((T)2, R::mul(l2, (T)nbr));
            T t = R::mul(a, c);
            t = R::add(t, R::mul(l2, s));
            T x = R::sub(t, pv);
            if (node) {
                x = bnd_math<T, MB>(x, uprev, nbr, mi, tab, M, l, gb, vb);
#pragma unroll
                for (int b = 0; b < MB; b++) {
                    gst[(int64_t)b * Nb + rank] = gb[b];
                    vst[(int64_t)b * Nb + rank] = vb[b];
                }
                ub[rank] = x;  // u^{n+2} at the node: read back as u^n two steps later
            }
            out[p] = x;
        }
    }
    // the last block adds the source and records the receivers
    __shared__ int last;
    __shared__ __align__(16) Ctl<T> cb;
    __syncthreads();
    if (threadIdx.x == 0) {
        __threadfence();
        last = atomicAdd(ticket, 1u) == gridDim.x - 1;
    }
    __syncthreads();
    if (last) {
        __threadfence();
        src_rcv_block<T>(out, ub, ctl, src_mode, 0, 0, cb);
        if (threadIdx.x == 0) *ticket = 0u;
    }
}

// node count of every 32-entry group of the shell list
__global__ void k_shell_wcount(const uint8_t *__restrict__ nmask, int64_t n, int64_t *__restrict__ cnt)
{
    const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const bool node = i < n && __popc(nmask[i]) < 6;
    const unsigned b = __ballot_sync(0xffffffffu, node);
    if ((threadIdx.x & 31) == 0 && i < n) cnt[i >> 5] = __popc(b);
}

// ------------------------------------------------------------------ host side
static PFN_cuTensorMapEncodeTiled_v12000 tb_encode_fn()
{
    static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
    if (!fn) {
        cudaDriverEntryPointQueryResult q;
        void *p = nullptr;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
            q == cudaDriverEntryPointSuccess)
            fn = (PFN_cuTensorMapEncodeTiled_v12000)p;
    }
    return fn;
}

static bool tb_map(CUtensorMap *m, CUtensorMapDataType dt, size_t esize, void *base, const Grid &g, int bx, int by,
                   int xpad = 0)
{
    auto fn = tb_encode_fn();
    if (!fn) return false;
    cuuint64_t dims[3] = {(cuuint64_t)(g.pitch + xpad), (cuuint64_t)(g.ny + 2), (cuuint64_t)(g.lnz + 2)};
    cuuint64_t strides[2] = {(cuuint64_t)(g.pitch * esize), (cuuint64_t)(g.plane * esize)};
    cuuint32_t box[3] = {(cuuint32_t)bx, (cuuint32_t)by, 1};
    cuuint32_t es[3] = {1, 1, 1};
    return fn(m, dt, 3, base, dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
              CU_TENSOR_MAP_L2_PROMOTION_L2_128B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

static constexpr int kTbTY = 32, kTbSU = 4, kTbSP = 4;

struct TwoStepPlan {
    CUtensorMap umap[4], pmap[4], kmap;
    int tiles_x, tiles_y, grid, smem;
    void *list = nullptr;  // shell positions (uint32 or int64), ascending
    uint8_t *nmask = nullptr;  // per shell entry: inside face neighbours (bits x-1, x+1, y-1, y+1, z-1, z+1)
    int64_t *wbase = nullptr;  // [n/32 + 1] boundary nodes before each 32-entry group of the list
    int64_t n_nodes = 0;       // boundary nodes in the list
    int64_t n_shell = 0;
    int64_t sh_lo = 0, sh_hi = 0;  // list range of the local planes [1, lnz-1) (slab interior)
    int64_t *src = nullptr;  // [7] the source's star, -1 = none
    bool idx64 = false;
    unsigned int *work = nullptr;  // [2] dynamic unit counter, CTAs done
};

// dynamic unit scheduling in k_volume2 (RAFD_TB_DYNAMIC = 0 never, 1 always,
// unset: units of >= 24 planes).  Measured (same box, A/B, ms per launch): C4 3.415 -> 3.277,
// 3072x1024x704 7.70 -> 6.47, C5 2048x1536x2560 34.9 -> 28.9: under the static
// order a CTA that falls behind processes its tiles rounds after their
// neighbours, whose shared halo rows have then left L2.
static int tb_dynamic_env()
{
    static int v = -2;
    if (v == -2) {
        const char *e = getenv("RAFD_TB_DYNAMIC");
        v = e ? (atoi(e) != 0) : -1;
    }
    return v;
}
static constexpr int kTbDynMinChunk = 24;  // unset: dynamic for units of >= 24 planes (small rooms stay static)

template <typename T>
cudaError_t twostep_plan_create(const Grid &g, void *const u[4], uint8_t *K_alloc, const uint8_t *K, bool idx64,
                                int nsm, cudaStream_t s, void **plan_out, int64_t *n_shell)
{
    using G = TbGeom<T, kTbTY, kTbSU, kTbSP>;
    auto *pl = new TwoStepPlan();
    const CUtensorMapDataType dt = sizeof(T) == 4 ? CU_TENSOR_MAP_DATA_TYPE_FLOAT32 : CU_TENSOR_MAP_DATA_TYPE_FLOAT64;
    bool ok = true;
    for (int k = 0; k < 4; k++) {
        ok = ok && tb_map(&pl->umap[k], dt, sizeof(T), u[k], g, G::UROW, G::UR);
        ok = ok && tb_map(&pl->pmap[k], dt, sizeof(T), u[k], g, G::TX, G::PR);
    }
    ok = ok && tb_map(&pl->kmap, CU_TENSOR_MAP_DATA_TYPE_UINT8, 1, K_alloc, g, G::KROW, G::PR, k_shift(g));
    if (!ok) {
        delete pl;
        return cudaErrorNotSupported;
    }
    pl->tiles_x = (g.nx + G::TXO - 1) / G::TXO;
    pl->tiles_y = (g.ny + kTbTY - 1) / kTbTY;
    pl->smem = G::SMEM;
    pl->idx64 = idx64;
    auto kern = k_volume2<T, kTbTY, kTbSU, kTbSP, false>;
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, pl->smem);
    if (e == cudaSuccess)
        e = cudaFuncSetAttribute(k_volume2<T, kTbTY, kTbSU, kTbSP, true>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                 pl->smem);
    int occ = 0;
    if (e == cudaSuccess) e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kern, G::NT, pl->smem);
    if (e == cudaSuccess && occ < 1) e = cudaErrorInvalidConfiguration;
    pl->grid = nsm * std::max(occ, 1);
    // the shell list
    const int64_t rows = (int64_t)g.lnz * g.ny;
    int64_t *cnt = nullptr, *off = nullptr;
    void *tmp = nullptr;
    size_t tb = 0;
    if (e == cudaSuccess) e = dev_alloc((void **)&cnt, (size_t)(rows + 1) * 8);
    if (e == cudaSuccess) e = dev_alloc((void **)&off, (size_t)(rows + 1) * 8);
    if (e == cudaSuccess) e = cudaMemsetAsync(cnt, 0, (size_t)(rows + 1) * 8, s);
    if (e == cudaSuccess) e = launch_shell_counts(g, K, cnt, s);
    if (e == cudaSuccess) e = exclusive_scan_rows64(cnt, off, rows + 1, nullptr, &tb, s);
    if (e == cudaSuccess) e = dev_alloc((void **)&tmp, tb ? tb : 16);
    if (e == cudaSuccess) e = exclusive_scan_rows64(cnt, off, rows + 1, tmp, &tb, s);
    int64_t n = 0;
    if (e == cudaSuccess) e = cudaMemcpyAsync(&n, off + rows, 8, cudaMemcpyDeviceToHost, s);
    if (e == cudaSuccess && g.lnz >= 2) e = cudaMemcpyAsync(&pl->sh_lo, off + g.ny, 8, cudaMemcpyDeviceToHost, s);
    if (e == cudaSuccess && g.lnz >= 2)
        e = cudaMemcpyAsync(&pl->sh_hi, off + (int64_t)(g.lnz - 1) * g.ny, 8, cudaMemcpyDeviceToHost, s);
    if (e == cudaSuccess) e = cudaStreamSynchronize(s);
    if (e == cudaSuccess) e = dev_alloc((void **)&pl->list, (size_t)std::max<int64_t>(n, 1) * (idx64 ? 8 : 4));
    if (e == cudaSuccess) e = dev_alloc((void **)&pl->nmask, (size_t)std::max<int64_t>(n, 1));
    if (e == cudaSuccess && n > 0) e = launch_shell_compact(g, K, off, idx64, pl->list, pl->nmask, s);
    // node count per 32-entry group, scanned (the fused shell + boundary kernel)
    const int64_t ngr = (n + 31) / 32;
    int64_t *wcnt = nullptr;
    void *wtmp = nullptr;
    size_t wtb = 0;
    if (e == cudaSuccess) e = dev_alloc((void **)&wcnt, (size_t)(ngr + 1) * 8);
    if (e == cudaSuccess) e = dev_alloc((void **)&pl->wbase, (size_t)(ngr + 1) * 8);
    if (e == cudaSuccess) e = cudaMemsetAsync(wcnt, 0, (size_t)(ngr + 1) * 8, s);
    if (e == cudaSuccess && n > 0) {
        k_shell_wcount<<<(unsigned)((n + 255) / 256), 256, 0, s>>>(pl->nmask, n, wcnt);
        e = cudaGetLastError();
    }
    if (e == cudaSuccess) e = exclusive_scan_rows64(wcnt, pl->wbase, ngr + 1, nullptr, &wtb, s);
    if (e == cudaSuccess) e = dev_alloc(&wtmp, wtb ? wtb : 16);
    if (e == cudaSuccess) e = exclusive_scan_rows64(wcnt, pl->wbase, ngr + 1, wtmp, &wtb, s);
    if (e == cudaSuccess) e = cudaMemcpyAsync(&pl->n_nodes, pl->wbase + ngr, 8, cudaMemcpyDeviceToHost, s);
    if (e == cudaSuccess) e = cudaStreamSynchronize(s);
    if (wcnt) dev_free(wcnt);
    if (wtmp) dev_free(wtmp);
    if (e == cudaSuccess) e = dev_alloc((void **)&pl->work, 2 * sizeof(unsigned int));
    if (e == cudaSuccess) e = cudaMemsetAsync(pl->work, 0, 2 * sizeof(unsigned int), s);
    if (e == cudaSuccess) e = dev_alloc((void **)&pl->src, 7 * 8);
    if (e == cudaSuccess) e = cudaMemsetAsync(pl->src, 0xff, 7 * 8, s);
    if (e == cudaSuccess) e = cudaStreamSynchronize(s);
    if (cnt) dev_free(cnt);
    if (off) dev_free(off);
    if (tmp) dev_free(tmp);
    pl->n_shell = n;
    if (e != cudaSuccess) {
        if (pl->list) dev_free(pl->list);
        if (pl->nmask) dev_free(pl->nmask);
        if (pl->wbase) dev_free(pl->wbase);
        if (pl->src) dev_free(pl->src);
        if (pl->work) dev_free(pl->work);
        delete pl;
        return e;
    }
    *n_shell = n;
    *plan_out = pl;
    return cudaSuccess;
}

void twostep_plan_destroy(void *plan)
{
    auto *pl = (TwoStepPlan *)plan;
    if (!pl) return;
    if (pl->list) dev_free(pl->list);
    if (pl->nmask) dev_free(pl->nmask);
    if (pl->wbase) dev_free(pl->wbase);
    if (pl->src) dev_free(pl->src);
    if (pl->work) dev_free(pl->work);
    delete pl;
}

int64_t twostep_shell_nodes(const void *plan) { return plan ? ((const TwoStepPlan *)plan)->n_nodes : -1; }

cudaError_t twostep_set_source(void *plan, int64_t pos, const Grid &g)
{
    auto *pl = (TwoStepPlan *)plan;
    int64_t h[7];
    for (int k = 0; k < 7; k++) h[k] = -1;
    if (pos >= 0) {
        const int64_t d[7] = {0, -1, 1, -g.pitch, g.pitch, -g.plane, g.plane};
        for (int k = 0; k < 7; k++) h[k] = pos + d[k];
    }
    return cudaMemcpy(pl->src, h, sizeof h, cudaMemcpyHostToDevice);
}

// Cap on the planes one unit marches (RAFD_TB_ZCHUNK_MAX, 0 = none; default
// 256).  Measured with dynamic scheduling, ms per launch: C5 (chunk 366
// uncapped) 28.4 -> 24.3 at 256; C4 (118) and 3072x1024x704 (235) unchanged;
// 64-176 cost C4 / 3072x1024x704 1-2 % (the z ring restarts per unit).
static int tb_zchunk_cap()
{
    static int v = -1;
    if (v < 0) {
        const char *e = getenv("RAFD_TB_ZCHUNK_MAX");
        v = e ? std::max(0, atoi(e)) : 256;
    }
    return v;
}

static int tb_choose_zchunk(int nz, int tiles, int grid)
{
    long best = -1;
    const int cap = tb_zchunk_cap();
    int best_c = cap ? std::min(nz, cap) : nz;
    for (int n = 1; n <= nz; n++) {
        const int c = (nz + n - 1) / n;
        if (cap && c > cap) continue;
        const long units = (long)tiles * ((nz + c - 1) / c);
        const long rounds = (units + grid - 1) / grid;
        const long cost = rounds * (c + 4);  // +4: the z ring recomputed / re-read per chunk
        if (best < 0 || cost < best) {
            best = cost;
            best_c = c;
        }
        if (c == 1) break;
    }
    return best_c;
}

template <typename T>
cudaError_t launch_volume2(const void *plan, const Grid &g, int cur_buf, int prev_buf, T *out1, T *out2,
                           double lambda, cudaStream_t s, int z_lo, int z_hi)
{
    using G = TbGeom<T, kTbTY, kTbSU, kTbSP>;
    const auto *pl = (const TwoStepPlan *)plan;
    if (z_hi < 0) z_hi = g.lnz;
    if (z_hi <= z_lo) return cudaSuccess;
    const T l2 = (T)(lambda * lambda);
    const int tiles = pl->tiles_x * pl->tiles_y;
    const int zc = tb_choose_zchunk(z_hi - z_lo, tiles, pl->grid);
    const long units = (long)tiles * ((z_hi - z_lo + zc - 1) / zc);
    const int grid = (int)std::min<long>(pl->grid, units);
    const int env = tb_dynamic_env();
    if (env == 1 || (env < 0 && zc >= kTbDynMinChunk))
        k_volume2<T, kTbTY, kTbSU, kTbSP, true><<<grid, G::NT, pl->smem, s>>>(
            pl->umap[cur_buf], pl->pmap[prev_buf], pl->kmap, out1, out2, g, l2, z_lo, z_hi, zc, pl->tiles_x,
            pl->tiles_y, pl->work);
    else
        k_volume2<T, kTbTY, kTbSU, kTbSP, false><<<grid, G::NT, pl->smem, s>>>(
            pl->umap[cur_buf], pl->pmap[prev_buf], pl->kmap, out1, out2, g, l2, z_lo, z_hi, zc, pl->tiles_x,
            pl->tiles_y, nullptr);
    return cudaGetLastError();
}

template <typename T>
cudaError_t launch_shell(const void *plan, const Grid &g, const T *u1, const T *u0, const uint8_t *K, T *out,
                         double lambda, cudaStream_t s, bool interior)
{
    const auto *pl = (const TwoStepPlan *)plan;
    const T l2 = (T)(lambda * lambda);
    if (interior && g.lnz < 3) return cudaSuccess;
    const int64_t lo = interior ? pl->sh_lo : 0, cnt = interior ? pl->sh_hi - pl->sh_lo : pl->n_shell;
    const int zp_lo = interior ? 2 : 1, zp_hi = interior ? g.lnz : g.lnz + 1;
    const int64_t n = cnt + 7;
    const unsigned blocks = (unsigned)((n + 255) / 256);
    if (pl->idx64)
        k_shell<T, int64_t><<<blocks, 256, 0, s>>>((const int64_t *)pl->list + lo, pl->nmask + lo, cnt, pl->src, u1, u0, K, out, g,
                                                   l2, zp_lo, zp_hi);
    else
        k_shell<T, uint32_t><<<blocks, 256, 0, s>>>((const uint32_t *)pl->list + lo, pl->nmask + lo, cnt, pl->src, u1, u0, K, out, g,
                                                    l2, zp_lo, zp_hi);
    return cudaGetLastError();
}

static constexpr int kShellEnt = 1;  // entries per thread of k_shell_bnd

template <typename T, int MB>
static cudaError_t launch_sb(const TwoStepPlan *pl, const Grid &g, const T *u1, const T *u0, const uint8_t *K,
                             T *out, T l2, T l, const uint8_t *matb, T *ub, T *gst, T *vst, int64_t Nb, const T *tab,
                             int M, Ctl<T> *ctl, unsigned int *ticket, cudaStream_t s, int64_t lo, int64_t hi,
                             int zp_lo, int zp_hi, int src_mode)
{
    constexpr int ENT = kShellEnt;
    const int64_t n = hi - (lo & ~(int64_t)31);
    const unsigned blocks = (unsigned)((n + 7 + 256 * ENT - 1) / (256 * ENT));
    if (pl->idx64)
        k_shell_bnd<T, MB, int64_t, ENT><<<blocks, 256, 0, s>>>((const int64_t *)pl->list, pl->nmask, pl->wbase, lo, hi,
                                                               pl->src, u1, u0, K, out, g, l2, l, matb, ub, gst, vst,
                                                               Nb, tab, M, ctl, ticket, zp_lo, zp_hi, src_mode);
    else
        k_shell_bnd<T, MB, uint32_t, ENT><<<blocks, 256, 0, s>>>((const uint32_t *)pl->list, pl->nmask, pl->wbase, lo,
                                                                hi, pl->src, u1, u0, K, out, g, l2, l, matb, ub, gst,
                                                                vst, Nb, tab, M, ctl, ticket, zp_lo, zp_hi, src_mode);
    return cudaGetLastError();
}

template <typename T>
cudaError_t launch_shell_bnd(const void *plan, const Grid &g, const T *u1, const T *u0, const uint8_t *K, T *out,
                             double lambda, int MB, const uint8_t *matb, T *ub, T *gst, T *vst, int64_t Nb,
                             const T *tab, int M, Ctl<T> *ctl, unsigned int *ticket, cudaStream_t s, bool interior,
                             int src_mode)
{
    const auto *pl = (const TwoStepPlan *)plan;
    const T l2 = (T)(lambda * lambda), l = (T)lambda;
    if (interior && g.lnz < 3) return cudaSuccess;
    const int64_t lo = interior ? pl->sh_lo : 0, hi = interior ? pl->sh_hi : pl->n_shell;
    const int zp_lo = interior ? 2 : 1, zp_hi = interior ? g.lnz : g.lnz + 1;
#define RAFD_SB(k) \
    case k:        \
        return launch_sb<T, k>(pl, g, u1, u0, K, out, l2, l, matb, ub, gst, vst, Nb, tab, M, ctl, ticket, s, lo, hi, zp_lo, zp_hi, src_mode);
    switch (MB) {
        RAFD_SB(0)
        RAFD_SB(1)
        RAFD_SB(2)
        RAFD_SB(3)
        RAFD_SB(4)
        RAFD_SB(5)
        RAFD_SB(6)
        RAFD_SB(7)
        RAFD_SB(8)
        default: return cudaErrorInvalidValue;
    }
#undef RAFD_SB
}

#define RAFD_TB_INST(T)                                                                                            \
    template cudaError_t twostep_plan_create<T>(const Grid &, void *const[4], uint8_t *, const uint8_t *, bool, int, \
                                                cudaStream_t, void **, int64_t *);                                  \
    template cudaError_t launch_volume2<T>(const void *, const Grid &, int, int, T *, T *, double, cudaStream_t,    \
                                           int, int);                                                               \
    template cudaError_t launch_shell<T>(const void *, const Grid &, const T *, const T *, const uint8_t *, T *,     \
                                         double, cudaStream_t, bool);                                                 \
    template cudaError_t launch_shell_bnd<T>(const void *, const Grid &, const T *, const T *, const uint8_t *, T *, \
                                             double, int, const uint8_t *, T *, T *, T *, int64_t, const T *, int,   \
                                             Ctl<T> *, unsigned int *, cudaStream_t, bool, int);
RAFD_TB_INST(float)
RAFD_TB_INST(double)
#undef RAFD_TB_INST

}  // namespace rafd
