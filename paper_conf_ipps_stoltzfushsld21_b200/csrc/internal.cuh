// internal.cuh -- shared definitions of the CUDA library (not part of the ABI).
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

#include <algorithm>
#include <string>
#include <vector>

#include "../../include/rafd.h"

namespace rafd {

// ------------------------------------------------------------------ arithmetic
// Correctly rounded single operations (no FMA contraction), DESIGN.md §4.
template <typename T> struct rn;
template <> struct rn<float> {
    static __device__ __forceinline__ float add(float a, float b) { return __fadd_rn(a, b); }
    static __device__ __forceinline__ float sub(float a, float b) { return __fsub_rn(a, b); }
    static __device__ __forceinline__ float mul(float a, float b) { return __fmul_rn(a, b); }
    static __device__ __forceinline__ float div(float a, float b) { return __fdiv_rn(a, b); }
};
template <> struct rn<double> {
    static __device__ __forceinline__ double add(double a, double b) { return __dadd_rn(a, b); }
    static __device__ __forceinline__ double sub(double a, double b) { return __dsub_rn(a, b); }
    static __device__ __forceinline__ double mul(double a, double b) { return __dmul_rn(a, b); }
    static __device__ __forceinline__ double div(double a, double b) { return __ddiv_rn(a, b); }
};

// ------------------------------------------------------------------ grid layout
// Padded grid in HBM: (lnz+2) planes x (ny+2) rows x pitch
// elements.  Room voxel (x, y, zl) (zl slab-local, 0..lnz-1) lives at
//   (zl+1)*plane + (y+1)*pitch + xo + x
// with xo = 128/sizeof(T) so every interior row starts on a 128-byte line
// (a tile's u^{n-1} reads and u+ stores then cover whole sectors, never a
// sector shared with the neighbouring tile); the x halo cells are xo-1 and
// xo+nx; pitch is a multiple of 128 bytes.  The uint8 K grid uses the same
// element indexing, shifted by k_shift(g) bytes from its allocation so that
// element xo of every row is 16-byte aligned (TMA box origin).
struct Grid {
    int32_t nx, ny, lnz;
    int32_t xo;
    int64_t pitch, plane, total;
};
static inline __host__ __device__ int k_shift(const Grid &g) { return (16 - g.xo % 16) % 16; }

// Device control block for the per-step source / receivers (read by the
// src/rcv kernel so that CUDA graphs never need re-capturing).
template <typename T> struct Ctl {
    int64_t n;          // step counter (index into sig)
    int64_t rec_count;  // samples recorded since the last read
    int64_t rec_cap;    // capacity of rec (rows)
    T *rec;             // [rec_cap][nrcv]
    const T *sig;       // [sig_len]
    int64_t sig_len;
    int64_t src_pos;    // padded index or -1
    int64_t src_node;   // boundary-node index of the source voxel or -1 (its u_b slot is updated too)
    int32_t nrcv;
    int32_t pad_;
    const int64_t *rcv_pos;  // [nrcv] padded indices
};

struct KernelTimes {
    double volume_ms = 0, boundary_ms = 0, other_ms = 0, shell_ms = 0;
    int64_t volume_n = 0, boundary_n = 0, other_n = 0, shell_n = 0;
};

// ------------------------------------------------------------------ device memory (devmem.cu)
// cached = true: the block may come from / return to the library's cache
cudaError_t dev_alloc(void **p, size_t bytes, bool cached = true);
void dev_free(void *p);
bool dev_cache_enabled();
void dev_cache_trim(int dev, size_t keep);

// ------------------------------------------------------------------ launchers
// (each returns cudaGetLastError() of its launch)
// Arguments of the fused volume+boundary kernel (seg_first is set by the plan).
template <typename T> struct FusedArgs {
    const int32_t *seg_first;
    const uint8_t *matb;
    T *g, *v;
    const T *tab;
    int M, MB;
    int64_t Nb;
    T l;
    int scheme;      // 0: Listing 2 volume; 1: Listing 1 single kernel; 2: Listing 6 naive FI
    T beta1;         // Listing 1 admittance
    T loss1, loss2;  // Listing 6 constants
    const uint8_t *occ;  // [lnz+2][tiles] tile-plane occupancy (set by the plan), or nullptr
    // halo push: byte offsets from an output address to the
    // same voxel in a neighbour's ghost plane (peer memory); 0 = no mirror
    int64_t mirror[2];
    // dynamic unit scheduling (set by the plan): [2] atomic unit counter and
    // CTAs-done count, reset by the last CTA; nullptr = static round-robin
    unsigned int *work;
    // units that hold an inside voxel (set by the plan for whole-room launches of
    // non-cuboid rooms): chunk << 16 | tile, ascending; nullptr = every unit
    const uint32_t *ulist;
    int nulist;
};

// plan == nullptr selects the one-thread-per-voxel v0 kernel (A/B reference);
// fa->scheme != 0 selects a single-kernel scheme (then no boundary kernel runs);
// cur_idx = which field buffer holds u^n, prev_idx u^{n-1} (default cur_idx ^ 1,
// in place; selects the TMA maps);
// fa != nullptr (and a fused plan) applies the boundary update in the same pass.
template <typename T>
cudaError_t launch_volume(const Grid &g, const T *cur, T *nxt, const uint8_t *K, double lambda,
                          int z_lo, int z_hi, cudaStream_t s, const void *plan, int cur_idx,
                          const FusedArgs<T> *fa = nullptr, int prev_idx = -1);
cudaError_t volume_plan_fuse(void *plan, const Grid &g, const uint8_t *K, int64_t Nb, cudaStream_t s);
bool volume_plan_fused(const void *plan);
cudaError_t volume_plan_occupancy(void *plan, const Grid &g, const uint8_t *K, cudaStream_t s);
template <typename T>
cudaError_t volume_plan_create(const Grid &g, void *const u[4], uint8_t *K, int nsm, void **plan);
void volume_plan_destroy(void *plan);
void volume_plan_adopt_occupancy(void *dst_plan, void *src_plan);
// temporal blocking (twostep.cu): the two-step volume kernel over the four
// field buffers (cur_buf = u^n, prev_buf = u^{n-1} -> out1 = u^{n+1}, out2 =
// u^{n+2}) and the shell recompute of u^{n+2} (list built by the plan)
template <typename T>
cudaError_t twostep_plan_create(const Grid &g, void *const u[4], uint8_t *K_alloc, const uint8_t *K, bool idx64,
                                int nsm, cudaStream_t s, void **plan, int64_t *n_shell);
void twostep_plan_destroy(void *plan);
cudaError_t twostep_set_source(void *plan, int64_t pos, const Grid &g);
template <typename T>
cudaError_t launch_volume2(const void *plan, const Grid &g, int cur_buf, int prev_buf, T *out1, T *out2,
                           double lambda, cudaStream_t s, int z_lo = 0, int z_hi = -1);
// interior: only the local planes [1, lnz-1) of a z slab (its edge planes are
// recomputed whole by the single-step kernel after the halo exchange)
template <typename T>
cudaError_t launch_shell(const void *plan, const Grid &g, const T *u1, const T *u0, const uint8_t *K, T *out,
                         double lambda, cudaStream_t s, bool interior = false);
// the shell fused with the step-(n+2) boundary update and the source /
// receivers (src_mode as k_boundary's); the list's node entries must be
// exactly the handle's nodes (twostep_shell_nodes(plan) == Nb).  interior: a
// slab's interior planes only (list range [sh_lo, sh_hi), nodes
// [n_first_plane, n_last_start))
template <typename T>
cudaError_t launch_shell_bnd(const void *plan, const Grid &g, const T *u1, const T *u0, const uint8_t *K, T *out,
                             double lambda, int MB, const uint8_t *matb, T *ub, T *gst, T *vst, int64_t Nb,
                             const T *tab, int M, Ctl<T> *ctl, unsigned int *ticket, cudaStream_t s,
                             bool interior = false, int src_mode = 3);
int64_t twostep_shell_nodes(const void *plan);
template <typename T>
cudaError_t launch_boundary(int MB, bool idx64, const void *bpos, const uint8_t *Kb,
                            const uint8_t *matb, int64_t i_lo, int64_t i_hi, int64_t Nb, T *unext,
                            T *ub, T *g, T *v, const T *tab, const T *tab_host, int M, double lambda,
                            cudaStream_t s, int64_t mirror0 = 0, int64_t mirror1 = 0, Ctl<T> *ctl = nullptr,
                            unsigned int *ticket = nullptr, int src_mode = 3);
template <typename T>
cudaError_t launch_src_rcv(T *unext, T *ub, Ctl<T> *ctl, cudaStream_t s, int mode = 3, int64_t mirror0 = 0,
                           int64_t mirror1 = 0);
cudaError_t launch_find_node(const void *bpos, bool idx64, int64_t Nb, int64_t pos, int64_t *out,
                             cudaStream_t s);

// classification: flags -> K (in place, bit 7 trick), counts, compaction
cudaError_t launch_scatter_mask(const Grid &g, const uint8_t *mask_chunk, int zp0, int nzc,
                                uint8_t *K, cudaStream_t s);
cudaError_t launch_scatter_mask_bits(const Grid &g, const uint32_t *bits, int rw, int zp0, int nzc, uint8_t *K,
                                     cudaStream_t s);
// host side of the bit-packed mask upload (maskpack.cu)
int pack_threads();
void pack_mask_rows(const uint8_t *mask, int64_t nrows, int nx, uint32_t *out, int rw, int nthreads);
cudaError_t launch_count_k(const Grid &g, uint8_t *K, cudaStream_t s);
cudaError_t launch_finish_k(const Grid &g, uint8_t *K, unsigned long long *hist8,
                            cudaStream_t s);
cudaError_t launch_row_counts64(const Grid &g, const uint8_t *K, int64_t *counts, cudaStream_t s);
cudaError_t launch_compact(const Grid &g, const uint8_t *K, const int64_t *row_off, int64_t zglob0,
                           int32_t ny_glob, int32_t nx_glob, bool idx64, void *bpos,
                           int64_t *bidx, uint8_t *Kb, cudaStream_t s);
// shell voxels of the two-step kernel (inside, and itself or a face neighbour
// with K < 6): per-row counts and the ascending list of padded positions
cudaError_t launch_shell_counts(const Grid &g, const uint8_t *K, int64_t *counts, cudaStream_t s);
cudaError_t launch_shell_compact(const Grid &g, const uint8_t *K, const int64_t *off, bool idx64, void *list,
                                 uint8_t *nmask, cudaStream_t s);
cudaError_t launch_gather_mat(const uint8_t *matmap_chunk, int64_t canon0, const int64_t *bidx,
                              int64_t i_lo, int64_t i_hi, uint8_t *matb, int M,
                              unsigned int *bad_flag, cudaStream_t s);
cudaError_t exclusive_scan_rows64(const int64_t *counts, int64_t *row_off, int64_t n, void *tmp,
                                  size_t *tmp_bytes, cudaStream_t s);

// fields in / out (canonical <-> padded), chunked over planes
template <typename T>
cudaError_t launch_field_in(const Grid &g, const T *src_chunk, int z0, int nzc, const uint8_t *K,
                            T *dst, cudaStream_t s);
template <typename T>
cudaError_t launch_field_out(const Grid &g, const T *src, int z0, int nzc, T *dst_chunk,
                             cudaStream_t s);
template <typename T>
cudaError_t launch_gather_ub(const void *bpos, bool idx64, int64_t Nb, const T *u, T *ub,
                             cudaStream_t s);
template <typename T>
cudaError_t launch_energy(const Grid &g, const T *un1, const T *un, const uint8_t *K, double *acc,
                          cudaStream_t s);
template <typename T>
cudaError_t launch_energy_bnd(const uint8_t *Kb, const uint8_t *matb, int64_t Nb, int MB,
                              const T *v, const T *gst, const double *DF, int M, double lambda,
                              double *acc, cudaStream_t s);

}  // namespace rafd
