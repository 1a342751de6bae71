/*
 * oracle.c -- plain, slow, sequential CPU oracle for GPU-ICD (Sabne et al., PPoPP'17).
 *
 * TEST INFRASTRUCTURE ONLY (see oracle.h).  C99, IEEE double, single thread.
 * Every function cites the PAPER.md passage (P:line) or DESIGN.md reading it follows.
 * Nothing here is shared with the CUDA path.
 */
#include "oracle.h"

#include <math.h>
#include <stdlib.h>
#include <string.h>
#include <pthread.h>

#define ORC_PI 3.14159265358979323846
#define ORC_EPS 1e-9 /* channel-index guard, reading R5 */

/* ------------------------------------------------------------------------------------
 * System matrix.  P:83-87: each view theta is one sinogram column; the sensors that see a
 * voxel at a view are those whose rays cross it.  Reading R4: A_ij = area(strip_i ∩
 * pixel_j) / dchannel (strip-integral model for a parallel-beam detector of pitch dc).
 * ---------------------------------------------------------------------------------- */

typedef struct { double x, y; } pt;

/* keep the part of polygon `in` (n vertices) where sgn*(x*c + y*s - t) >= 0 */
static int clip_halfplane(const pt* in, int n, pt* out, double c, double s, double t, double sgn)
{
    int m = 0;
    for (int i = 0; i < n; ++i) {
        pt a = in[i], b = in[(i + 1) % n];
        double da = sgn * (a.x * c + a.y * s - t);
        double db = sgn * (b.x * c + b.y * s - t);
        if (da >= 0) out[m++] = a;
        if ((da >= 0) != (db >= 0)) {
            double r = da / (da - db);
            pt q;
            q.x = a.x + r * (b.x - a.x);
            q.y = a.y + r * (b.y - a.y);
            out[m++] = q;
        }
    }
    return m;
}

double orc_strip_pixel_area(double cx, double cy, double d, double c, double s,
                            double tlo, double thi)
{
    pt sq[4], p1[8], p2[12];
    double h = 0.5 * d;
    /* area is translation invariant: clip in pixel-centred coordinates so the shoelace sums
     * stay O(d^2) instead of O(|centre|^2) (no cancellation for thin slivers far off-axis) */
    const double tc = cx * c + cy * s;
    tlo -= tc;
    thi -= tc;
    sq[0].x = -h; sq[0].y = -h;
    sq[1].x = +h; sq[1].y = -h;
    sq[2].x = +h; sq[2].y = +h;
    sq[3].x = -h; sq[3].y = +h;
    int n1 = clip_halfplane(sq, 4, p1, c, s, tlo, +1.0); /* x*c+y*s >= tlo */
    if (n1 < 3) return 0.0;
    int n2 = clip_halfplane(p1, n1, p2, c, s, thi, -1.0); /* x*c+y*s <= thi */
    if (n2 < 3) return 0.0;
    double a = 0.0; /* shoelace */
    for (int i = 0; i < n2; ++i) {
        pt u = p2[i], v = p2[(i + 1) % n2];
        a += u.x * v.y - v.x * u.y;
    }
    return fabs(0.5 * a);
}

/* P:273 "720 uniformly distributed views between 0 and 180 degrees" -> theta_k = k*pi/V. */
double orc_view_angle(const orc_geom* g, int k)
{
    if (g->angles) return g->angles[k];
    return (double)k * ORC_PI / (double)g->nviews;
}

int orc_sysmatrix_column(const orc_geom* g, int ix, int iy, int K,
                         int32_t* first, int32_t* count, double* vals)
{
    const double d = g->dxy, dc = g->dchannel;
    const int M = g->nchannels;
    /* pixel centres, row-major [iy][ix], image centred on the rotation axis (reading R4) */
    const double cx = ((double)ix - 0.5 * (double)(g->nx - 1)) * d;
    const double cy = ((double)iy - 0.5 * (double)(g->ny - 1)) * d;
    const double t0 = -0.5 * (double)M * dc + g->center_offset * dc;
    int maxc = 0;
    for (int k = 0; k < g->nviews; ++k) {
        double th = orc_view_angle(g, k);
        double c = cos(th), s = sin(th);
        double tj = cx * c + cy * s;
        double h2 = 0.5 * d * (fabs(c) + fabs(s)); /* half-width of the pixel's shadow */
        /* channels whose strip can meet the shadow [tj-h2, tj+h2] (reading R5) */
        int f = (int)floor((tj - h2 - t0) / dc + ORC_EPS);
        int l = (int)ceil((tj + h2 - t0) / dc - ORC_EPS) - 1;
        if (f < 0) f = 0;
        if (l > M - 1) l = M - 1;
        int n = l - f + 1;
        if (n < 0) n = 0;
        if (n > maxc) maxc = n;
        first[k] = (n > 0) ? f : 0;
        count[k] = (n > K) ? K : n;
        for (int i = 0; i < K; ++i) vals[(int64_t)k * K + i] = 0.0;
        for (int i = 0; i < n && i < K; ++i) {
            double lo = t0 + (double)(f + i) * dc, hi = lo + dc;
            vals[(int64_t)k * K + i] = orc_strip_pixel_area(cx, cy, d, c, s, lo, hi) / dc;
        }
    }
    return maxc;
}

int orc_sysmatrix_build(const orc_geom* g, int K, int32_t* first, int32_t* count, double* vals)
{
    int maxc = 0;
    const int V = g->nviews;
    for (int iy = 0; iy < g->ny; ++iy)
        for (int ix = 0; ix < g->nx; ++ix) {
            int64_t j = (int64_t)iy * g->nx + ix;
            int m = orc_sysmatrix_column(g, ix, iy, K, first + j * V, count + j * V,
                                         vals + j * V * K);
            if (m > maxc) maxc = m;
        }
    return maxc;
}

/* newAEntry = (unsigned char)(AEntry / max_voxel * 255 + 0.5), per-voxel max
 * stored for dequantisation (reading R6: scale then round half up). */
double orc_quantize_column(const double* vals, const int32_t* count, int nviews, int K,
                           uint8_t* codes)
{
    double amax = 0.0;
    for (int k = 0; k < nviews; ++k)
        for (int i = 0; i < count[k]; ++i)
            if (vals[(int64_t)k * K + i] > amax) amax = vals[(int64_t)k * K + i];
    for (int k = 0; k < nviews; ++k)
        for (int i = 0; i < K; ++i) {
            double a = vals[(int64_t)k * K + i];
            codes[(int64_t)k * K + i] =
                (i < count[k] && amax > 0.0) ? (uint8_t)floor(a / amax * 255.0 + 0.5) : 0;
        }
    return amax;
}

/* ------------------------------------------------------------------------------------
 * Prior.  P:107-109 (Alg1:7) calls func(v, theta1, theta2, neighbours of v) and says only
 * that it is "computationally inexpensive".  Reading R1: q-GGMRF potential with the
 * symmetric-bound quadratic surrogate; reading R2: 1/distance neighbour weights.
 * ---------------------------------------------------------------------------------- */
double orc_rho(double delta, const orc_prior* pr)
{
    double a = fabs(delta);
    if (a == 0.0) return 0.0;
    double u = pow(a / (pr->T * pr->sigma), pr->q - pr->p);
    return pow(a, pr->p) / (pr->p * pow(pr->sigma, pr->p)) * u / (1.0 + u);
}

/* phi(D) = rho'(D)/(2D) = |D|^(p-2)/(2 s^p) * u (q/p + u) / (1+u)^2 ; limit at D=0 (q=2). */
double orc_phi(double delta, const orc_prior* pr)
{
    double a = fabs(delta);
    double sp = pow(pr->sigma, pr->p);
    if (a == 0.0) {
        if (pr->q == pr->p) {
            /* u == 1 identically: phi = |D|^(p-2)/(2 s^p) * (q/p + 1)/4, finite only for p = 2 */
            if (pr->p < 2.0) return INFINITY;
            return (pr->q / pr->p + 1.0) / (8.0 * sp);
        }
        /* q > p: u -> 0 and lim_{D->0} = (q/p) / (2 s^p (T s)^(q-p)) for q = 2 (+inf for q < 2) */
        if (pr->q < 2.0) return INFINITY;
        return (pr->q / pr->p) / (2.0 * sp * pow(pr->T * pr->sigma, pr->q - pr->p));
    }
    double u = pow(a / (pr->T * pr->sigma), pr->q - pr->p);
    return pow(a, pr->p - 2.0) / (2.0 * sp) * u * (pr->q / pr->p + u) / ((1.0 + u) * (1.0 + u));
}

double orc_nbr_weight(int dx, int dy, int dz, int nbhd)
{
    int ax = abs(dx), ay = abs(dy), az = abs(dz);
    if (ax > 1 || ay > 1 || az > 1) return 0.0;
    int m = ax + ay + az;
    if (m == 0) return 0.0;
    if (nbhd == 8) {
        if (az != 0) return 0.0;
        double norm = 4.0 + 4.0 / sqrt(2.0);
        return (m == 1 ? 1.0 : 1.0 / sqrt(2.0)) / norm;
    }
    /* 26-neighbourhood: 6 faces (1), 12 edges (1/sqrt2), 8 corners (1/sqrt3) */
    double norm = 6.0 + 12.0 / sqrt(2.0) + 8.0 / sqrt(3.0);
    return (1.0 / sqrt((double)m)) / norm;
}

/* ------------------------------------------------------------------------------------
 * Alg. 1 with func = exact minimiser of the surrogate, clipped (reading R1, R3).
 * ---------------------------------------------------------------------------------- */
void orc_voxel_update(const orc_geom* g, const orc_prior* pr, int K,
                      const int32_t* col_first, const int32_t* col_count, const double* col_vals,
                      const double* w, double* x, double* e, int64_t j, int apply,
                      double* theta1_out, double* theta2_out, double* delta_out)
{
    const int nx = g->nx, ny = g->ny, nz = g->nz, V = g->nviews, M = g->nchannels;
    const int64_t plane = (int64_t)nx * ny;
    const int iz = (int)(j / plane);
    const int iy = (int)((j % plane) / nx);
    const int ix = (int)(j % nx);
    const double* ws = w + (int64_t)iz * V * M;
    double* es = e + (int64_t)iz * V * M;

    /* Alg1:1-6: theta1 = -sum w*A*e, theta2 = sum w*A^2 over (view, sensor) of the voxel */
    double theta1 = 0.0, theta2 = 0.0;
    for (int k = 0; k < V; ++k)
        for (int i = 0; i < col_count[k]; ++i) {
            int64_t idx = (int64_t)k * M + col_first[k] + i;
            double a = col_vals[(int64_t)k * K + i];
            theta1 += -ws[idx] * a * es[idx];
            theta2 += ws[idx] * a * a;
        }

    /* Alg1:7: delta = func(v, theta1, theta2, neighbours of v).  Surrogate coefficients
     * bt_r = b_jr * phi(v - x_r); minimiser u* = (theta2 v - theta1 + 2 sum bt_r x_r) /
     * (theta2 + 2 sum bt_r); clip at 0 (reading R3). */
    const double v = x[j];
    double num = theta2 * v - theta1, den = theta2;
    for (int dz = -1; dz <= 1; ++dz)
        for (int dy = -1; dy <= 1; ++dy)
            for (int dx = -1; dx <= 1; ++dx) {
                double b = orc_nbr_weight(dx, dy, dz, pr->nbhd);
                if (b == 0.0) continue;
                int rx = ix + dx, ry = iy + dy, rz = iz + dz;
                if (rx < 0 || rx >= nx || ry < 0 || ry >= ny || rz < 0 || rz >= nz) continue;
                double xr = x[((int64_t)rz * ny + ry) * nx + rx];
                double bt = b * orc_phi(v - xr, pr);
                num += 2.0 * bt * xr;
                den += 2.0 * bt;
            }
    double u = (den > 0.0) ? num / den : v;
    if (pr->positivity && u < 0.0) u = 0.0;
    double delta = u - v;

    if (apply) {
        x[j] = v + delta; /* Alg1:8 */
        for (int k = 0; k < V; ++k) /* Alg1:9-11: e -= A*delta */
            for (int i = 0; i < col_count[k]; ++i) {
                int64_t idx = (int64_t)k * M + col_first[k] + i;
                es[idx] -= col_vals[(int64_t)k * K + i] * delta;
            }
    }
    if (theta1_out) *theta1_out = theta1;
    if (theta2_out) *theta2_out = theta2;
    if (delta_out) *delta_out = delta;
}

/* splitmix64 (public-domain generator) for the random visiting order of P:115 */
static uint64_t splitmix64(uint64_t* s)
{
    uint64_t z = (*s += 0x9E3779B97F4A7C15ULL);
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
    return z ^ (z >> 31);
}

/* zero-skip predicate of P:115: the voxel and all of its neighbours are zero */
static int all_zero_nbhd(const orc_geom* g, int nbhd, const double* x, int64_t j)
{
    const int nx = g->nx, ny = g->ny, nz = g->nz;
    const int64_t plane = (int64_t)nx * ny;
    const int iz = (int)(j / plane), iy = (int)((j % plane) / nx), ix = (int)(j % nx);
    if (x[j] != 0.0) return 0;
    for (int dz = -1; dz <= 1; ++dz)
        for (int dy = -1; dy <= 1; ++dy)
            for (int dx = -1; dx <= 1; ++dx) {
                if (orc_nbr_weight(dx, dy, dz, nbhd) == 0.0) continue;
                int rx = ix + dx, ry = iy + dy, rz = iz + dz;
                if (rx < 0 || rx >= nx || ry < 0 || ry >= ny || rz < 0 || rz >= nz) continue;
                if (x[((int64_t)rz * ny + ry) * nx + rx] != 0.0) return 0;
            }
    return 1;
}

/* zero-skip in this 1-based sweep?  P:115 skips from the second sweep on (reading R9); with a
 * re-admission period P > 0 every P-th sweep runs without skipping, so a voxel frozen at 0 is
 * re-examined and a fixed point of the iteration is a fixed point of plain ICD (the MAP). */
static int skip_sweep(int zero_skip, int period, int sweep)
{
    return zero_skip && sweep > 1 && !(period > 0 && sweep % period == 0);
}

int64_t orc_icd_run(const orc_geom* g, const orc_prior* pr, int K,
                    const int32_t* first, const int32_t* count, const double* vals,
                    const double* w, double* x, double* e,
                    int n_equits, int first_sweep, uint64_t seed, int zero_skip, int zero_skip_period,
                    const int64_t* order, int64_t order_len,
                    double* dump, int64_t dump_cap, orc_stats* st)
{
    const int64_t plane = (int64_t)g->nx * g->ny;
    const int64_t nvox = plane * g->nz;
    const int V = g->nviews;
    int64_t ndump = 0;
    int64_t* perm = NULL;
    if (!order) {
        perm = (int64_t*)malloc(sizeof(int64_t) * (size_t)nvox);
        if (!perm) return -1;
    }
    for (int s = 0; s < n_equits; ++s) {
        int sweep = first_sweep + s; /* 1-based sweep number */
        const int64_t* seq;
        int64_t n;
        if (order) {
            seq = order;
            n = order_len;
        } else {
            /* fresh random permutation per sweep ("randomized order") */
            uint64_t st64 = seed ^ ((uint64_t)sweep * 0xD1B54A32D192ED03ULL);
            for (int64_t i = 0; i < nvox; ++i) perm[i] = i;
            for (int64_t i = nvox - 1; i > 0; --i) {
                int64_t r = (int64_t)(splitmix64(&st64) % (uint64_t)(i + 1));
                int64_t t = perm[i];
                perm[i] = perm[r];
                perm[r] = t;
            }
            seq = perm;
            n = nvox;
        }
        for (int64_t q = 0; q < n; ++q) {
            int64_t j = seq[q];
            if (skip_sweep(zero_skip, zero_skip_period, sweep) && all_zero_nbhd(g, pr->nbhd, x, j)) {
                if (st) st->skipped++;
                continue;
            }
            int64_t jj = j % plane; /* A is slice-invariant in parallel beam */
            double t1, t2, dl;
            orc_voxel_update(g, pr, K, first + jj * V, count + jj * V, vals + jj * V * K, w, x,
                             e, j, 1, &t1, &t2, &dl);
            if (st) {
                st->updates++;
                st->sum_abs_delta += fabs(dl);
            }
            if (dump && ndump < dump_cap) {
                dump[4 * ndump + 0] = (double)j;
                dump[4 * ndump + 1] = t1;
                dump[4 * ndump + 2] = t2;
                dump[4 * ndump + 3] = dl;
                ndump++;
            }
        }
    }
    free(perm);
    return ndump;
}

/* Sequential ICD in slice-parity halves (golden runs of 3-D volumes): per sweep,
 * for parity 0 then 1, every slice z of that parity runs one pass over its own voxels in a
 * fresh random order (splitmix64 Fisher-Yates seeded from (seed, sweep, z)).  Slices of one
 * parity share no sinogram entry (each slice has its own e, parallel beam) and no prior edge
 * (the 26-neighbourhood links z to z +- 1 only), so running them on several threads at once is
 * exactly the sequential ICD of their concatenated orders: an exact serialisation, not an
 * approximation.  POSIX threads pull slices from a shared counter. */
typedef struct {
    const orc_geom* g;
    const orc_prior* pr;
    int K;
    const int32_t *first, *count;
    const double *vals, *w;
    double *x, *e;
    uint64_t seed;
    int sweep, parity, skip;
    int next; /* next slice index of this parity to take (guarded by the mutex) */
    pthread_mutex_t mu;
    int64_t upd, skp;
    double sad;
    int fail;
} zpar_job;

static void zpar_slice(zpar_job* J, int z, int64_t* perm, int64_t* upd, int64_t* skp, double* sad)
{
    const orc_geom* g = J->g;
    const int64_t plane = (int64_t)g->nx * g->ny;
    uint64_t st64 = J->seed ^ ((uint64_t)J->sweep * 0xD1B54A32D192ED03ULL) ^ ((uint64_t)(z + 1) * 0x9E3779B97F4A7C15ULL);
    for (int64_t i = 0; i < plane; ++i) perm[i] = i;
    for (int64_t i = plane - 1; i > 0; --i) {
        int64_t r = (int64_t)(splitmix64(&st64) % (uint64_t)(i + 1));
        int64_t t = perm[i];
        perm[i] = perm[r];
        perm[r] = t;
    }
    for (int64_t q = 0; q < plane; ++q) {
        const int64_t jj = perm[q], j = (int64_t)z * plane + jj;
        if (J->skip && all_zero_nbhd(g, J->pr->nbhd, J->x, j)) {
            (*skp)++;
            continue;
        }
        double dl;
        orc_voxel_update(g, J->pr, J->K, J->first + jj * g->nviews, J->count + jj * g->nviews,
                         J->vals + jj * g->nviews * J->K, J->w, J->x, J->e, j, 1, NULL, NULL, &dl);
        (*upd)++;
        *sad += fabs(dl);
    }
}

static void* zpar_worker(void* arg)
{
    zpar_job* J = (zpar_job*)arg;
    const int64_t plane = (int64_t)J->g->nx * J->g->ny;
    int64_t* perm = (int64_t*)malloc(sizeof(int64_t) * (size_t)plane);
    int64_t upd = 0, skp = 0;
    double sad = 0.0;
    for (;;) {
        pthread_mutex_lock(&J->mu);
        const int z = J->next;
        J->next += 2;
        pthread_mutex_unlock(&J->mu);
        if (z >= J->g->nz || !perm) break;
        zpar_slice(J, z, perm, &upd, &skp, &sad);
    }
    pthread_mutex_lock(&J->mu);
    J->upd += upd;
    J->skp += skp;
    J->sad += sad;
    if (!perm) J->fail = 1;
    pthread_mutex_unlock(&J->mu);
    free(perm);
    return NULL;
}

int orc_icd_run_zpar(const orc_geom* g, const orc_prior* pr, int K, const int32_t* first,
                     const int32_t* count, const double* vals, const double* w, double* x,
                     double* e, int n_equits, int first_sweep, uint64_t seed, int zero_skip,
                     int zero_skip_period, int nthreads, orc_stats* st)
{
    zpar_job J;
    memset(&J, 0, sizeof(J));
    J.g = g; J.pr = pr; J.K = K; J.first = first; J.count = count; J.vals = vals; J.w = w;
    J.x = x; J.e = e; J.seed = seed;
    pthread_mutex_init(&J.mu, NULL);
    if (nthreads < 1) nthreads = 1;
    if (nthreads > 256) nthreads = 256;
    pthread_t th[256];
    for (int s = 0; s < n_equits && !J.fail; ++s) {
        J.sweep = first_sweep + s;
        J.skip = skip_sweep(zero_skip, zero_skip_period, J.sweep);
        for (int parity = 0; parity < 2; ++parity) {
            J.parity = parity;
            J.next = parity;
            int started = 0;
            for (int t = 0; t < nthreads; ++t)
                if (pthread_create(&th[t], NULL, zpar_worker, &J) == 0) ++started;
            if (started == 0) zpar_worker(&J);
            for (int t = 0; t < started; ++t) pthread_join(th[t], NULL);
        }
    }
    pthread_mutex_destroy(&J.mu);
    if (st) {
        st->updates += J.upd;
        st->skipped += J.skp;
        st->sum_abs_delta += J.sad;
    }
    return J.fail ? -1 : 0;
}

void orc_error_sinogram(const orc_geom* g, int K, const int32_t* first, const int32_t* count,
                        const double* vals, const double* y, const double* x, double* e)
{
    const int V = g->nviews, M = g->nchannels;
    const int64_t plane = (int64_t)g->nx * g->ny;
    memcpy(e, y, sizeof(double) * (size_t)g->nz * V * M);
    for (int z = 0; z < g->nz; ++z)
        for (int64_t jj = 0; jj < plane; ++jj) {
            double xv = x[z * plane + jj];
            if (xv == 0.0) continue;
            for (int k = 0; k < V; ++k)
                for (int i = 0; i < count[jj * V + k]; ++i)
                    e[((int64_t)z * V + k) * M + first[jj * V + k] + i] -=
                        vals[(jj * V + k) * K + i] * xv;
        }
}

double orc_cost(const orc_geom* g, const orc_prior* pr, int K, const int32_t* first,
                const int32_t* count, const double* vals, const double* y, const double* w,
                const double* x)
{
    const int nx = g->nx, ny = g->ny, nz = g->nz, V = g->nviews, M = g->nchannels;
    const int64_t nsino = (int64_t)nz * V * M;
    double* e = (double*)malloc(sizeof(double) * (size_t)nsino);
    if (!e) return NAN;
    orc_error_sinogram(g, K, first, count, vals, y, x, e);
    double data = 0.0;
    for (int64_t i = 0; i < nsino; ++i) data += 0.5 * w[i] * e[i] * e[i];
    free(e);
    double prior = 0.0; /* each unordered pair {j, r} once: count it from the lower index */
    for (int iz = 0; iz < nz; ++iz)
        for (int iy = 0; iy < ny; ++iy)
            for (int ix = 0; ix < nx; ++ix) {
                int64_t j = ((int64_t)iz * ny + iy) * nx + ix;
                for (int dz = -1; dz <= 1; ++dz)
                    for (int dy = -1; dy <= 1; ++dy)
                        for (int dx = -1; dx <= 1; ++dx) {
                            double b = orc_nbr_weight(dx, dy, dz, pr->nbhd);
                            if (b == 0.0) continue;
                            int rx = ix + dx, ry = iy + dy, rz = iz + dz;
                            if (rx < 0 || rx >= nx || ry < 0 || ry >= ny || rz < 0 || rz >= nz)
                                continue;
                            int64_t r = ((int64_t)rz * ny + ry) * nx + rx;
                            if (r <= j) continue;
                            prior += b * orc_rho(x[j] - x[r], pr);
                        }
            }
    return data + prior;
}

double orc_rmse_hu(const double* a, const double* b, int64_t n, double mu_water)
{
    double s = 0.0;
    for (int64_t i = 0; i < n; ++i) s += (a[i] - b[i]) * (a[i] - b[i]);
    return 1000.0 * sqrt(s / (double)n) / mu_water;
}
