/*
 * orc.h -- the CPU ORACLE for the room-acoustics FDTD step.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and the
 * cpu_baseline / --impl reference legs of bench.py may load liborc.so.  The
 * product library (include/rafd.h, paper_conf_ipps_stoltzfushsld21_b200/csrc)
 * never includes, links or calls anything in this directory, and this
 * directory never includes anything from the product: the two share no code,
 * headers, tables or constants.
 *
 * What it computes (citations are PAPER.md line numbers = the paper text in
 * /root/reference/PAPER.md, with the section / listing they fall in):
 *
 *   classification   PAPER.md:306-323 (Sec. II-B): nbrs[idx] = number of the 6
 *                    face neighbours lying inside; 0 for outside points.
 *                    Boundary point <=> 0 < K < 6 (Listing 1 rule,
 *                    PAPER.md:280-291); boundaryIndices PAPER.md:390-393.
 *   volume kernel    PAPER.md:349-357 (Listing 2, kernel 1).
 *   FI-MM boundary   PAPER.md:371-381 (Listing 3).
 *   FD-MM boundary   PAPER.md:415-442 (Listing 4), typos read as in DESIGN.md
 *                    (readings R6, R7).
 *   iteration        PAPER.md:850-889 (Listing 5, "the two kernels are
 *                    executed iteratively").
 *
 * Arithmetic: working precision T (float or double) for every operation the
 * listings perform, in the listings' left-to-right evaluation order, no FMA
 * contraction (built with -ffp-contract=off), IEEE division.  The FD
 * coefficients BI, DI, beta are derived from the physical (D, E, F, beta0)
 * in double (reading R5) and rounded once to T.
 *
 * The same oracle is also built with orc_abi.c into librafd_oracle.so, which
 * exports the product's C-ABI names (rafd_create, rafd_step, ...) with the same
 * semantics for whole rooms; tests/test_oracle_abi.py drives
 * it through the product's own Python binding.
 *
 * Pins: see tests/test_oracle_*.py.  Every function below is pinned there
 * against something other than itself (closed forms, Table II counts,
 * energy invariants, brute-force dense matrices, exact reflection
 * coefficients) -- see DESIGN.md "Oracle pins".
 */
#ifndef ORC_H
#define ORC_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define ORC_OK 0
#define ORC_E_INVAL -1
#define ORC_E_UNSTABLE -2
#define ORC_E_NONPASSIVE -3
#define ORC_E_OUTSIDE -4
#define ORC_E_MATERIAL -5
#define ORC_E_NOMEM -6

typedef struct orc_room orc_room;

typedef struct orc_desc {
    int32_t nx, ny, nz;          /* room (mask) dims; the oracle adds a 1-voxel outside halo */
    const uint8_t *mask;         /* [nz][ny][nx], x fastest; nonzero = inside            */
    const uint8_t *matmap;       /* [nz][ny][nx] material id, read at boundary nodes; NULL => 0 */
    double lambda;               /* Courant number l ("l", "l2")           */
    int32_t precision;           /* 32 or 64                                               */
    int32_t n_materials;         /* M >= 1                                                 */
    int32_t n_branches;          /* MB: 0 => FI-MM (Listing 3), >= 1 => FD-MM (Listing 4)  */
    const double *beta0;         /* [M]  FI admittance (MB=0) / instantaneous part (MB>0)  */
    const double *D, *E, *F;     /* [M*MB] row-major [m][b]; ignored when MB = 0           */
} orc_desc;

typedef struct orc_info {
    int64_t n_mask, n_inside, n_boundary;
    int64_t k_hist[7];
    int64_t isolated;
    int64_t steps;
    int32_t precision, n_materials, n_branches;
} orc_info;

int  orc_create(const orc_desc *d, orc_room **out);
/* Test-only: Listing-4 tables used verbatim (rounded to T), no passivity and no
 * stability (lambda) check.
 * beta[M], BI/D/DI/F [M*MB].  Used to show that inconsistent tables are unstable. */
int  orc_create_raw(const orc_desc *d, const double *beta, const double *BI,
                    const double *D, const double *DI, const double *F, orc_room **out);
void orc_destroy(orc_room *r);

int  orc_set_source(orc_room *r, int32_t x, int32_t y, int32_t z, const double *sig, int64_t len);
int  orc_set_receivers(orc_room *r, int32_t n, const int32_t *xyz);
/* Initial state.  u_prev/u_curr: T-typed [nz][ny][nx] (NULL => keep); values at
 * outside voxels are forced to +0.  v, g: T-typed [MB][Nb] (NULL => keep). */
int  orc_set_state(orc_room *r, const void *u_prev, const void *u_curr, const void *v, const void *g);
int  orc_step(orc_room *r, int64_t nsteps);
/* Checkpoint / resume: the step counter indexes the source signal. */
int  orc_set_step(orc_room *r, int64_t n);
/* Single-kernel schemes of the paper: 0 = Listings 2-4 (default),
 * 1 = Listing 1 (n_materials = 1, MB = 0, beta = beta0[0]),
 * 2 = Listing 6 naive FI (constants loss1, loss2, reading R17). */
int  orc_set_scheme(orc_room *r, int32_t scheme, double loss1, double loss2);
int  orc_read_receivers(orc_room *r, double *out, int64_t cap, int64_t *n_written);
/* Fields as T-typed [nz][ny][nx]: u^n (curr) and u^{n-1} (prev).  NULL => skip. */
int  orc_read_field(orc_room *r, void *u_curr, void *u_prev);
int  orc_read_branch_state(orc_room *r, void *v, void *g);
int  orc_get_classification(orc_room *r, uint8_t *K, int64_t *bidx, uint8_t *Kb, uint8_t *matb);
int  orc_get_info(orc_room *r, orc_info *info);
/* Discrete energy H^{n+1/2} (reading R11), in double. */
int  orc_energy(orc_room *r, double *H);
const char *orc_last_error(void);
/* OpenMP threads for the volume / boundary loops (process-wide); results are
 * independent of the count. */
int  orc_set_threads(int32_t n);
int32_t orc_get_threads(void);

#ifdef __cplusplus
}
#endif
#endif
