/*
 * orc_abi.c -- the CPU oracle behind the product's C-ABI names (SURVEY.md §8(b):
 * "librafd_oracle.so exports the same names and semantics (CPU, device/NCCL
 * fields ignored), implemented independently").  TEST INFRASTRUCTURE ONLY (see
 * orc.h): built with orc.c into oracle/librafd_oracle.so, so that the product's
 * own Python binding (paper_conf_ipps_stoltzfushsld21_b200/rafd.py, pointed at
 * this library) can drive the oracle through exactly the calls a user makes
 * (tests/test_oracle_abi.py).
 *
 * The descriptor structs below are this file's own declarations of the ABI's
 * layout (plain C structs with the same members in the same order); nothing is
 * included from the product, and the product includes nothing from here.
 * Whole rooms only: a slab descriptor (nranks > 1) is refused with STATE, as
 * are the device-side calls (IPC, halo push, step groups).  Temporal blocking
 * and profiling are accepted and change nothing: the oracle always steps
 * Listings 2-4 one step at a time, and the CUDA path is bitwise equal to that.
 */
#include <math.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#include "orc.h"

#define RAFD_OK 0
#define RAFD_E_INVAL -1
#define RAFD_E_STATE -9

typedef struct rafd_materials {
    int32_t n_materials, n_branches;
    const double *beta0;
    const double *D, *E, *F;
} rafd_materials;

typedef struct rafd_room_desc {
    int32_t nx, ny, nz;
    const uint8_t *mask;
    const uint8_t *matmap;
    double lambda;
    int32_t precision;
    const rafd_materials *mat;
    int32_t device;
    void *cuda_stream;
    int32_t rank, nranks;
    const uint8_t *nccl_id;
    int32_t z_begin, z_end;
    int32_t mask_z0;
    int32_t scheme;
    double loss1, loss2;
} rafd_room_desc;

typedef struct rafd_info {
    int64_t n_mask, n_inside, n_boundary;
    int64_t k_hist[7];
    int64_t isolated, steps;
    int64_t bytes_per_step, volume_bytes, boundary_bytes, device_bytes;
    int32_t precision, n_materials, n_branches;
    int32_t z_begin, z_end;
    int32_t pitch, fused, scheme, steps_per_sweep, reserved_;
    int64_t n_shell;
} rafd_info;

typedef struct rafd_kernel_times {
    double volume_ms, boundary_ms, other_ms;
    int64_t volume_launches, boundary_launches, other_launches;
    double shell_ms;
    int64_t shell_launches;
} rafd_kernel_times;

typedef struct rafd_room {
    orc_room *o;
    int32_t nx, ny, nz, precision, M, MB, scheme, tb;
} rafd_room;

static _Thread_local char g_abi_err[256];
static int abi_fail(int code, const char *msg)
{
    snprintf(g_abi_err, sizeof g_abi_err, "%s", msg);
    return code;
}
static int pass(int rc)
{
    if (rc) snprintf(g_abi_err, sizeof g_abi_err, "%s", orc_last_error());
    return rc; /* the oracle's codes are the ABI's codes (-1 .. -6) */
}

int rafd_create(const rafd_room_desc *d, rafd_room **out)
{
    if (!out) return abi_fail(RAFD_E_INVAL, "null out");
    *out = NULL;
    if (!d || !d->mat) return abi_fail(RAFD_E_INVAL, "null descriptor or materials");
    if (d->nranks > 1) return abi_fail(RAFD_E_STATE, "the oracle holds whole rooms (nranks <= 1)");
    if (d->mask_z0 != 0) return abi_fail(RAFD_E_INVAL, "the oracle reads the whole mask (mask_z0 = 0)");
    orc_desc od;
    memset(&od, 0, sizeof od);
    od.nx = d->nx;
    od.ny = d->ny;
    od.nz = d->nz;
    od.mask = d->mask;
    od.matmap = d->matmap;
    od.lambda = d->lambda;
    od.precision = d->precision;
    od.n_materials = d->mat->n_materials;
    od.n_branches = d->mat->n_branches;
    od.beta0 = d->mat->beta0;
    od.D = d->mat->D;
    od.E = d->mat->E;
    od.F = d->mat->F;
    orc_room *o = NULL;
    int rc = orc_create(&od, &o);
    if (rc) return pass(rc);
    if (d->scheme != 0 && (rc = orc_set_scheme(o, d->scheme, d->loss1, d->loss2))) {
        orc_destroy(o);
        return pass(rc);
    }
    rafd_room *r = calloc(1, sizeof *r);
    if (!r) {
        orc_destroy(o);
        return abi_fail(-6, "out of memory");
    }
    r->o = o;
    r->nx = d->nx;
    r->ny = d->ny;
    r->nz = d->nz;
    r->precision = d->precision;
    r->M = d->mat->n_materials;
    r->MB = d->mat->n_branches;
    r->scheme = d->scheme;
    r->tb = 1;
    *out = r;
    return RAFD_OK;
}

void rafd_destroy(rafd_room *r)
{
    if (!r) return;
    orc_destroy(r->o);
    free(r);
}

#define NEED(r) \
    if (!(r)) return abi_fail(RAFD_E_INVAL, "null room")

int rafd_set_source(rafd_room *r, int32_t x, int32_t y, int32_t z, const double *sig, int64_t len)
{
    NEED(r);
    return pass(orc_set_source(r->o, x, y, z, sig, len));
}
int rafd_set_receivers(rafd_room *r, int32_t n, const int32_t *xyz)
{
    NEED(r);
    return pass(orc_set_receivers(r->o, n, xyz));
}
int rafd_set_state(rafd_room *r, const void *u_prev, const void *u_curr, const void *v, const void *g)
{
    NEED(r);
    return pass(orc_set_state(r->o, u_prev, u_curr, v, g));
}
int rafd_set_step(rafd_room *r, int64_t n)
{
    NEED(r);
    return pass(orc_set_step(r->o, n));
}
int rafd_step(rafd_room *r, int64_t nsteps)
{
    NEED(r);
    return pass(orc_step(r->o, nsteps));
}
int rafd_set_temporal_blocking(rafd_room *r, int32_t steps_per_sweep)
{
    NEED(r);
    if (steps_per_sweep != 1 && steps_per_sweep != 2) return abi_fail(RAFD_E_INVAL, "steps_per_sweep must be 1 or 2");
    if (steps_per_sweep == 2 && r->scheme != 0) return abi_fail(RAFD_E_STATE, "temporal blocking runs the two-kernel scheme");
    r->tb = steps_per_sweep;
    return RAFD_OK;
}
int rafd_synchronize(rafd_room *r)
{
    NEED(r);
    return RAFD_OK;
}
int rafd_read_receivers(rafd_room *r, double *out, int64_t cap, int64_t *n_written)
{
    NEED(r);
    return pass(orc_read_receivers(r->o, out, cap, n_written));
}
int rafd_read_field(rafd_room *r, void *u_curr, void *u_prev)
{
    NEED(r);
    return pass(orc_read_field(r->o, u_curr, u_prev));
}
int rafd_read_branch_state(rafd_room *r, void *v, void *g)
{
    NEED(r);
    return pass(orc_read_branch_state(r->o, v, g));
}
int rafd_get_classification(rafd_room *r, uint8_t *K, int64_t *bidx, uint8_t *Kb, uint8_t *matb)
{
    NEED(r);
    return pass(orc_get_classification(r->o, K, bidx, Kb, matb));
}
int rafd_get_info(rafd_room *r, rafd_info *info)
{
    NEED(r);
    if (!info) return abi_fail(RAFD_E_INVAL, "null info");
    orc_info oi;
    int rc = orc_get_info(r->o, &oi);
    if (rc) return pass(rc);
    memset(info, 0, sizeof *info);
    info->n_mask = oi.n_mask;
    info->n_inside = oi.n_inside;
    info->n_boundary = oi.n_boundary;
    for (int k = 0; k < 7; k++) info->k_hist[k] = oi.k_hist[k];
    info->isolated = oi.isolated;
    info->steps = oi.steps;
    /* the algorithmic bytes of SURVEY.md §8(d): N_mask + 3s N_in + Nb (6 + 3s + 4s MB) */
    const int64_t s = r->precision / 8;
    info->volume_bytes = oi.n_mask + 3 * s * oi.n_inside;
    info->boundary_bytes = oi.n_boundary * (6 + 3 * s + 4 * s * r->MB);
    info->bytes_per_step = info->volume_bytes + info->boundary_bytes;
    info->precision = r->precision;
    info->n_materials = r->M;
    info->n_branches = r->MB;
    info->z_begin = 0;
    info->z_end = r->nz;
    info->pitch = r->nx + 2;
    info->scheme = r->scheme;
    info->steps_per_sweep = r->tb;
    return RAFD_OK;
}
int rafd_energy(rafd_room *r, double *H)
{
    NEED(r);
    return pass(orc_energy(r->o, H));
}
int rafd_set_profiling(rafd_room *r, int on)
{
    (void)on;
    NEED(r);
    return RAFD_OK;
}
int rafd_get_kernel_times(rafd_room *r, rafd_kernel_times *t)
{
    NEED(r);
    if (!t) return abi_fail(RAFD_E_INVAL, "null times");
    memset(t, 0, sizeof *t);
    return RAFD_OK;
}
int64_t rafd_launch_count(rafd_room *r)
{
    (void)r;
    return 0;
}

/* device-side and multi-process calls: not in the oracle */
int rafd_step_group(rafd_room **rooms, int32_t n, int64_t nsteps)
{
    (void)rooms, (void)n, (void)nsteps;
    return abi_fail(RAFD_E_STATE, "the oracle holds whole rooms (no slab groups)");
}
int rafd_ipc_handle(rafd_room *r, uint8_t *blob)
{
    (void)r, (void)blob;
    return abi_fail(RAFD_E_STATE, "no IPC in the oracle");
}
int rafd_ipc_connect(rafd_room *r, const uint8_t *lower, const uint8_t *upper)
{
    (void)r, (void)lower, (void)upper;
    return abi_fail(RAFD_E_STATE, "no IPC in the oracle");
}
int rafd_set_halo_push(rafd_room *r, int32_t on)
{
    (void)r;
    return on ? abi_fail(RAFD_E_STATE, "no halo in the oracle") : RAFD_OK;
}
int rafd_release_cached_memory(int32_t device)
{
    return device < 0 ? abi_fail(RAFD_E_INVAL, "device must be >= 0") : RAFD_OK;
}
int rafd_nccl_unique_id(uint8_t *id128)
{
    (void)id128;
    return abi_fail(-8, "no NCCL in the oracle");
}

/* the slab plan of SURVEY.md §8(e): z planes split by the prefix sum of the
 * per-plane cost c(z) = N_mask(z) + 3s N_in(z) + (6 + 3s + 4s MB) Nb(z), each cut
 * at the closer of the two planes around k/nranks of the total */
int rafd_slab_plan(int32_t nx, int32_t ny, int32_t nz, const uint8_t *mask, int32_t precision, int32_t n_branches,
                   int32_t nranks, int32_t *z_begin, int32_t *z_end)
{
    if (!mask || !z_begin || !z_end || nx < 1 || ny < 1 || nz < 1 || nranks < 1 || nranks > nz)
        return abi_fail(RAFD_E_INVAL, "bad slab-plan arguments");
    if (precision != 32 && precision != 64) return abi_fail(RAFD_E_INVAL, "precision must be 32 or 64");
    const double s = precision / 8;
    double *pre = calloc((size_t)nz + 1, sizeof(double));
    if (!pre) return abi_fail(-6, "out of memory");
    for (int32_t z = 0; z < nz; z++) {
        int64_t nin = 0, nb = 0;
        for (int32_t y = 0; y < ny; y++)
            for (int32_t x = 0; x < nx; x++) {
                if (!mask[((int64_t)z * ny + y) * nx + x]) continue;
                int k = 0;
                const int32_t dx[6] = {-1, 1, 0, 0, 0, 0}, dy[6] = {0, 0, -1, 1, 0, 0}, dz[6] = {0, 0, 0, 0, -1, 1};
                for (int j = 0; j < 6; j++) {
                    const int32_t a = x + dx[j], b = y + dy[j], c = z + dz[j];
                    if (a >= 0 && b >= 0 && c >= 0 && a < nx && b < ny && c < nz && mask[((int64_t)c * ny + b) * nx + a])
                        k++;
                }
                if (k > 0) nin++;
                if (k > 0 && k < 6) nb++;
            }
        pre[z + 1] = pre[z] + ((double)nx * ny + 3.0 * s * nin + (6.0 + 3.0 * s + 4.0 * s * n_branches) * nb);
    }
    int32_t prev = 0;
    for (int32_t k = 0; k < nranks; k++) {
        z_begin[k] = prev;
        int32_t e = nz;
        if (k < nranks - 1) {
            const double t = pre[nz] * (k + 1) / nranks;
            e = 0;
            while (e <= nz && pre[e] < t) e++; /* first e with pre[e] >= t */
            if (e > 0 && fabs(pre[e - 1] - t) <= fabs(pre[e] - t)) e--;
            if (e < prev + 1) e = prev + 1;
            if (e > nz - (nranks - 1 - k)) e = nz - (nranks - 1 - k);
        }
        z_end[k] = e;
        prev = e;
    }
    free(pre);
    return RAFD_OK;
}

const char *rafd_last_error(void) { return g_abi_err; }
const char *rafd_strerror(int code)
{
    switch (code) {
        case 0: return "ok";
        case -1: return "invalid argument";
        case -2: return "unstable Courant number (lambda^2 > 1/3)";
        case -3: return "non-passive boundary material";
        case -4: return "position outside the room";
        case -5: return "material id out of range";
        case -6: return "out of memory";
        case -7: return "CUDA error";
        case -8: return "NCCL error";
        case -9: return "invalid state";
        default: return "unknown error";
    }
}
int rafd_version(void) { return 1; }
