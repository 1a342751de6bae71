/* PSV-ICD: the paper's multi-core CPU comparison system (Alg. 2), built for
 * SURVEY 8(f) NEXT-4 so the GPU path can be set beside a parallel CPU ICD on the box's own
 * host cores (the paper's 4.43x GPU-ICD / PSV-ICD headline, is context only).
 *
 * NOT the product and NOT the oracle: a tuned-for-CPU float implementation.  It shares no code
 * with the CUDA path (csrc/) or with oracle/oracle.c; it takes the system matrix as plain arrays
 * (first channel, count, K values per (voxel, view)) from its caller.
 *
 * Alg. 2, in the paper's order:
 *   1   create SVs: s x s tiles of every slice (reading R13), per SV and view the band of
 *       channels its voxels touch (the SVB's row, Fig. 2 / P:121-123);
 *   4-9 iteration 1: all SVs; even iterations: the top `frac` of SVs by their last update amount
 *       (sum |delta|); odd iterations: a random `frac` of them (Alg. 2 uses 20 %);
 *   10  the selected SVs are processed in parallel on host threads (dynamic distribution, one SV
 *       per claim);
 *   11-13 create the weight SVB and the error SVB (copies of the band), keep SVB_e';
 *   14-15 update every voxel of the SV sequentially (Alg. 1) in a random order, from and
 *       into the SVB; zero-skip with the re-admission of reading R9 (iterations 1 + kP,
 *       random subsets, run without it);
 *   16-19 delta SVB = SVB_e' - SVB_e, and under one lock e <- e - delta SVB.
 * The SVB copy is taken under the same lock (the paper does not say; without it the copy would
 * race with another thread's write-back).  Voxel values of neighbouring SVs are read and written
 * with relaxed atomics (concurrent SVs may be adjacent, as in Alg. 2: no colouring).
 *
 * func (Alg1:7) is reading R1 (q-GGMRF, symmetric-bound surrogate), neighbours reading R2,
 * positivity R3; written here from DESIGN.md's formulas. */
#include "psvicd.h"

#include <math.h>
#include <pthread.h>
#include <stdlib.h>
#include <string.h>
#include <time.h>

typedef struct {
    int ix0, iy0, w, h;      /* tile origin and size (clipped at the image edge) */
    int bmax;                /* widest band row (channels) */
    int32_t* bstart;         /* [V] first channel of the band */
    int32_t* bwidth;         /* [V] channels in the band */
    uint8_t* off;            /* [nv][V] voxel's first channel - band start */
    float* a;                /* [nv][V][4] values (zero past the voxel's count) */
} sv_t;

struct psv_handle {
    psv_geom g;
    psv_prior pr;
    int side, nsx, nsy, nsv; /* SVs per slice */
    sv_t* sv;
    float nbw[27];           /* neighbour weights (dz+1)*9 + (dy+1)*3 + dx+1 */
    float* amount;           /* [nz][nsv] sum |delta| of the last visit */
    int iter;                /* iterations done */
    double inv_Ts, c_phi, pq, qmp; /* prior constants */
};

static double now_s(void)
{
    struct timespec t;
    clock_gettime(CLOCK_MONOTONIC, &t);
    return t.tv_sec + 1e-9 * t.tv_nsec;
}

static uint64_t smix(uint64_t z)
{
    z += 0x9E3779B97F4A7C15ULL;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
    return z ^ (z >> 31);
}

/* reading R2: 1/distance weights over the 8- (2-D) or 26- (3-D) neighbourhood, sum 1 */
static void nbr_weights(int nbhd, float* out)
{
    double norm = nbhd == 8 ? 4.0 + 4.0 / sqrt(2.0) : 6.0 + 12.0 / sqrt(2.0) + 8.0 / sqrt(3.0);
    for (int dz = -1; dz <= 1; ++dz)
        for (int dy = -1; dy <= 1; ++dy)
            for (int dx = -1; dx <= 1; ++dx) {
                int m = abs(dx) + abs(dy) + abs(dz);
                double b = 0.0;
                if (m > 0 && !(nbhd == 8 && dz != 0)) b = 1.0 / sqrt((double)m) / norm;
                out[(dz + 1) * 9 + (dy + 1) * 3 + dx + 1] = (float)b;
            }
}

/* reading R1: phi(D) = rho'(D)/(2D) of the q-GGMRF potential, q = 2 */
static inline float phi(const psv_handle* h, float d)
{
    float a = fabsf(d);
    float u = h->qmp == 0.0 ? 1.f : (a == 0.f ? 0.f : powf(a * (float)h->inv_Ts, (float)h->qmp));
    float opu = 1.f + u;
    return (float)h->c_phi * ((float)h->pq + u) / (opu * opu);
}

static inline float ld_x(const float* p)
{
    uint32_t b = __atomic_load_n((const uint32_t*)p, __ATOMIC_RELAXED);
    float f;
    memcpy(&f, &b, 4);
    return f;
}
static inline void st_x(float* p, float v)
{
    uint32_t b;
    memcpy(&b, &v, 4);
    __atomic_store_n((uint32_t*)p, b, __ATOMIC_RELAXED);
}

int psv_create(const psv_geom* g, const psv_prior* pr, int K, const int32_t* first, const int32_t* count,
               const double* vals, int sv_side, psv_handle** out)
{
    if (!g || !pr || !first || !count || !vals || !out || sv_side < 1 || K < 1 || K > 4) return -1;
    if (pr->q != 2.0 || pr->p < 1.0 || pr->p > 2.0 || !(pr->sigma > 0) || (pr->nbhd != 8 && pr->nbhd != 26))
        return -1;
    *out = NULL;
    psv_handle* h = calloc(1, sizeof(*h));
    if (!h) return -2;
    h->g = *g;
    h->pr = *pr;
    h->side = sv_side;
    h->nsx = (g->nx + sv_side - 1) / sv_side;
    h->nsy = (g->ny + sv_side - 1) / sv_side;
    h->nsv = h->nsx * h->nsy;
    nbr_weights(pr->nbhd, h->nbw);
    /* phi = |D|^(p-2)/(2 s^p) u (q/p + u)/(1+u)^2 with u = |D/(Ts)|^(q-p); for q = 2,
     * |D|^(p-2) u = (Ts)^(p-2), so phi = c (q/p + u)/(1+u)^2, c = (Ts)^(p-2)/(2 s^p) */
    h->inv_Ts = 1.0 / (pr->T * pr->sigma);
    h->qmp = pr->q - pr->p;
    h->pq = pr->q / pr->p;
    h->c_phi = pow(pr->T * pr->sigma, pr->p - 2.0) / (2.0 * pow(pr->sigma, pr->p));
    h->sv = calloc(h->nsv, sizeof(sv_t));
    h->amount = calloc((size_t)h->nsv * g->nz, sizeof(float));
    if (!h->sv || !h->amount) {
        psv_destroy(h);
        return -2;
    }
    const int V = g->nviews;
    for (int s = 0; s < h->nsv; ++s) {
        sv_t* S = &h->sv[s];
        S->ix0 = (s % h->nsx) * sv_side;
        S->iy0 = (s / h->nsx) * sv_side;
        S->w = g->nx - S->ix0 < sv_side ? g->nx - S->ix0 : sv_side;
        S->h = g->ny - S->iy0 < sv_side ? g->ny - S->iy0 : sv_side;
        const int nv = S->w * S->h;
        S->bstart = malloc(sizeof(int32_t) * V);
        S->bwidth = malloc(sizeof(int32_t) * V);
        S->off = malloc((size_t)nv * V);
        S->a = calloc((size_t)nv * V * 4, sizeof(float));
        if (!S->bstart || !S->bwidth || !S->off || !S->a) {
            psv_destroy(h);
            return -2;
        }
        S->bmax = 0;
        for (int k = 0; k < V; ++k) {
            int lo = 1 << 30, hi = -1;
            for (int v = 0; v < nv; ++v) {
                int64_t j = (int64_t)(S->iy0 + v / S->w) * g->nx + S->ix0 + v % S->w;
                int f = first[j * V + k], c = count[j * V + k];
                if (c <= 0) continue;
                if (f < lo) lo = f;
                if (f + c > hi) hi = f + c;
            }
            if (hi < 0) lo = hi = 0;
            S->bstart[k] = lo;
            S->bwidth[k] = hi - lo;
            if (hi - lo > S->bmax) S->bmax = hi - lo;
            if (hi - lo > 255) {
                psv_destroy(h);
                return -1;
            }
            for (int v = 0; v < nv; ++v) {
                int64_t j = (int64_t)(S->iy0 + v / S->w) * g->nx + S->ix0 + v % S->w;
                int c = count[j * V + k];
                S->off[(size_t)v * V + k] = (uint8_t)(c > 0 ? first[j * V + k] - lo : 0);
                for (int i = 0; i < c && i < K; ++i)
                    S->a[((size_t)v * V + k) * 4 + i] = (float)vals[(j * V + k) * K + i];
            }
        }
    }
    *out = h;
    return 0;
}

void psv_destroy(psv_handle* h)
{
    if (!h) return;
    if (h->sv)
        for (int s = 0; s < h->nsv; ++s) {
            free(h->sv[s].bstart);
            free(h->sv[s].bwidth);
            free(h->sv[s].off);
            free(h->sv[s].a);
        }
    free(h->sv);
    free(h->amount);
    free(h);
}

typedef struct {
    psv_handle* h;
    const float* w;
    float* x;
    float* e;
    const int32_t* tasks; /* (slice * nsv + sv) */
    int ntasks;
    int next;             /* atomic claim counter (dynamic distribution) */
    int skip;             /* zero-skip active this iteration */
    int raster;           /* raster visiting order instead of random (tests) */
    uint64_t seed;
    pthread_mutex_t mu;   /* Alg2:17-19 */
    int64_t updates, skipped;
    double sad;
} job_t;

/* zero-skip (reading R9): x_j and every neighbour exactly zero */
static int all_zero(const psv_handle* h, const float* x, int ix, int iy, int iz)
{
    const int nx = h->g.nx, ny = h->g.ny, nz = h->g.nz;
    for (int dz = -1; dz <= 1; ++dz)
        for (int dy = -1; dy <= 1; ++dy)
            for (int dx = -1; dx <= 1; ++dx) {
                if ((dx | dy | dz) && h->nbw[(dz + 1) * 9 + (dy + 1) * 3 + dx + 1] == 0.f) continue;
                int rx = ix + dx, ry = iy + dy, rz = iz + dz;
                if (rx < 0 || rx >= nx || ry < 0 || ry >= ny || rz < 0 || rz >= nz) continue;
                if (ld_x(&x[((int64_t)rz * ny + ry) * nx + rx]) != 0.f) return 0;
            }
    return 1;
}

static void visit(job_t* J, int task, float* svb_e, float* svb_w, float* svb_e0, int* order, int64_t* upd,
                  int64_t* skp, double* sad)
{
    psv_handle* h = J->h;
    const int V = h->g.nviews, M = h->g.nchannels, nx = h->g.nx, ny = h->g.ny;
    const int iz = task / h->nsv, s = task % h->nsv;
    const sv_t* S = &h->sv[s];
    const int st = S->bmax + 4; /* SVB row stride (views x band, padded for the 4-wide records) */
    const int nv = S->w * S->h;
    const int64_t zoff = (int64_t)iz * V * M;

    /* Alg2:11-13: SVB_w, SVB_e and SVB_e' (under the e lock, see the header) */
    pthread_mutex_lock(&J->mu);
    for (int k = 0; k < V; ++k) {
        const float* er = J->e + zoff + (int64_t)k * M + S->bstart[k];
        const float* wr = J->w + zoff + (int64_t)k * M + S->bstart[k];
        float* be = svb_e + (size_t)k * st;
        float* bw = svb_w + (size_t)k * st;
        const int bw_k = S->bwidth[k];
        memcpy(be, er, sizeof(float) * bw_k);
        memcpy(bw, wr, sizeof(float) * bw_k);
        for (int c = bw_k; c < st; ++c) be[c] = bw[c] = 0.f;
    }
    pthread_mutex_unlock(&J->mu);
    memcpy(svb_e0, svb_e, sizeof(float) * (size_t)V * st);

    /* random visiting order (Fisher-Yates from a per-(seed, iteration, task) stream) */
    for (int v = 0; v < nv; ++v) order[v] = v;
    if (!J->raster) {
        uint64_t r = smix(J->seed ^ smix(((uint64_t)h->iter << 32) ^ (uint64_t)task));
        for (int v = nv - 1; v > 0; --v) {
            r = smix(r);
            int u = (int)(r % (uint64_t)(v + 1));
            int t = order[v];
            order[v] = order[u];
            order[u] = t;
        }
    }
    double amount = 0.0;
    for (int n = 0; n < nv; ++n) {
        const int v = order[n];
        const int ix = S->ix0 + v % S->w, iy = S->iy0 + v / S->w;
        float* xj = &J->x[((int64_t)iz * ny + iy) * nx + ix];
        if (J->skip && all_zero(h, J->x, ix, iy, iz)) {
            ++*skp;
            continue;
        }
        /* Alg1:3-6 from the SVBs */
        const uint8_t* of = S->off + (size_t)v * V;
        const float* a = S->a + (size_t)v * V * 4;
        float t1 = 0.f, t2 = 0.f;
        for (int k = 0; k < V; ++k) {
            const float* be = svb_e + (size_t)k * st + of[k];
            const float* bw = svb_w + (size_t)k * st + of[k];
            const float* ak = a + (size_t)k * 4;
            for (int c = 0; c < 4; ++c) {
                float wa = bw[c] * ak[c];
                t1 -= wa * be[c];
                t2 += wa * ak[c];
            }
        }
        /* Alg1:7 (reading R1): minimiser of the surrogate, clipped at 0 (R3) */
        const float xv = ld_x(xj);
        float num = t2 * xv - t1, den = t2;
        for (int dz = -1; dz <= 1; ++dz)
            for (int dy = -1; dy <= 1; ++dy)
                for (int dx = -1; dx <= 1; ++dx) {
                    float b = h->nbw[(dz + 1) * 9 + (dy + 1) * 3 + dx + 1];
                    if (b == 0.f) continue;
                    int rx = ix + dx, ry = iy + dy, rz = iz + dz;
                    if (rx < 0 || rx >= nx || ry < 0 || ry >= ny || rz < 0 || rz >= h->g.nz) continue;
                    float xr = ld_x(&J->x[((int64_t)rz * ny + ry) * nx + rx]);
                    float bt = b * phi(h, xv - xr);
                    num += 2.f * bt * xr;
                    den += 2.f * bt;
                }
        float u = den > 0.f ? num / den : xv;
        if (h->pr.positivity && u < 0.f) u = 0.f;
        const float d = u - xv;
        ++*upd;
        if (d == 0.f) continue;
        st_x(xj, u); /* Alg1:8 */
        amount += fabsf(d);
        for (int k = 0; k < V; ++k) { /* Alg1:9-11 into the SVB */
            float* be = svb_e + (size_t)k * st + of[k];
            const float* ak = a + (size_t)k * 4;
            for (int c = 0; c < 4; ++c) be[c] -= ak[c] * d;
        }
    }
    *sad += amount;
    h->amount[task] = (float)amount;

    /* Alg2:16-19: delta SVB = SVB_e' - SVB_e; e <- e - delta SVB, under the lock */
    pthread_mutex_lock(&J->mu);
    for (int k = 0; k < V; ++k) {
        float* er = J->e + zoff + (int64_t)k * M + S->bstart[k];
        const float* be = svb_e + (size_t)k * st;
        const float* b0 = svb_e0 + (size_t)k * st;
        for (int c = 0; c < S->bwidth[k]; ++c) er[c] -= b0[c] - be[c];
    }
    pthread_mutex_unlock(&J->mu);
}

static void* worker(void* arg)
{
    job_t* J = arg;
    psv_handle* h = J->h;
    int bmax = 0, nvmax = 0;
    for (int s = 0; s < h->nsv; ++s) {
        if (h->sv[s].bmax > bmax) bmax = h->sv[s].bmax;
        if (h->sv[s].w * h->sv[s].h > nvmax) nvmax = h->sv[s].w * h->sv[s].h;
    }
    const size_t n = (size_t)h->g.nviews * (bmax + 4);
    float* buf = malloc(sizeof(float) * 3 * n);
    int* order = malloc(sizeof(int) * nvmax);
    int64_t upd = 0, skp = 0;
    double sad = 0.0;
    if (buf && order)
        for (;;) {
            int t = __atomic_fetch_add(&J->next, 1, __ATOMIC_RELAXED);
            if (t >= J->ntasks) break;
            visit(J, J->tasks[t], buf, buf + n, buf + 2 * n, order, &upd, &skp, &sad);
        }
    pthread_mutex_lock(&J->mu);
    J->updates += upd;
    J->skipped += skp;
    J->sad += sad;
    pthread_mutex_unlock(&J->mu);
    free(buf);
    free(order);
    return (buf && order) ? NULL : (void*)1;
}

static int cmp_desc(const void* a, const void* b)
{
    const float* fa = a;
    const float* fb = b;
    if (fa[0] != fb[0]) return fa[0] < fb[0] ? 1 : -1;
    return fa[1] < fb[1] ? -1 : (fa[1] > fb[1]);
}

int psv_iterate(psv_handle* h, const float* w, float* x, float* e, int n_iters, double frac, uint64_t seed,
                int zero_skip, int zero_skip_period, int nthreads, int raster, psv_stats* st)
{
    if (!h || !w || !x || !e || n_iters < 0 || !(frac > 0.0 && frac <= 1.0) || nthreads < 1) return -1;
    const int ntot = h->nsv * h->g.nz;
    int32_t* tasks = malloc(sizeof(int32_t) * ntot);
    float* keys = malloc(sizeof(float) * 2 * ntot);
    pthread_t* th = malloc(sizeof(pthread_t) * nthreads);
    if (!tasks || !keys || !th) {
        free(tasks);
        free(keys);
        free(th);
        return -2;
    }
    job_t J;
    memset(&J, 0, sizeof(J));
    J.h = h;
    J.w = w;
    J.x = x;
    J.e = e;
    J.tasks = tasks;
    J.seed = seed;
    J.raster = raster;
    pthread_mutex_init(&J.mu, NULL);
    const double t0 = now_s();
    int rc = 0;
    for (int it = 0; it < n_iters && rc == 0; ++it) {
        const int iter = ++h->iter;
        int n = 0;
        const int nsel = (int)ceil(frac * ntot);
        if (iter == 1) { /* Alg2:4-5 */
            for (int t = 0; t < ntot; ++t) tasks[n++] = t;
        } else if (iter % 2 == 0) { /* Alg2:6-7: top frac by update amount (ties: lower index) */
            for (int t = 0; t < ntot; ++t) {
                keys[2 * t] = h->amount[t];
                keys[2 * t + 1] = (float)t;
            }
            qsort(keys, ntot, 2 * sizeof(float), cmp_desc);
            for (int i = 0; i < nsel; ++i) tasks[n++] = (int32_t)keys[2 * i + 1];
        } else { /* Alg2:8-9: random frac (partial Fisher-Yates) */
            for (int t = 0; t < ntot; ++t) tasks[t] = t;
            uint64_t r = smix(seed ^ (0xA5A5ULL << 40) ^ (uint64_t)iter);
            for (int i = 0; i < nsel; ++i) {
                r = smix(r);
                int u = i + (int)(r % (uint64_t)(ntot - i));
                int32_t tt = tasks[i];
                tasks[i] = tasks[u];
                tasks[u] = tt;
            }
            n = nsel;
        }
        J.ntasks = n;
        J.next = 0;
        /* reading R9: iterations 1 + k P (odd: a random subset) run without zero-skip */
        J.skip = zero_skip && iter > 1 && !(zero_skip_period > 0 && (iter - 1) % zero_skip_period == 0);
        int started = 0;
        for (int t = 0; t < nthreads; ++t) /* Alg2:10 */
            if (pthread_create(&th[t], NULL, worker, &J) == 0) ++started;
        for (int t = 0; t < started; ++t) {
            void* res = NULL;
            pthread_join(th[t], &res);
            if (res) rc = -2;
        }
        if (started == 0) rc = -3;
    }
    const double t1 = now_s();
    pthread_mutex_destroy(&J.mu);
    if (st) {
        st->updates = J.updates;
        st->skipped = J.skipped;
        st->sum_abs_delta = J.sad;
        st->seconds = t1 - t0;
        st->iterations = h->iter;
    }
    free(tasks);
    free(keys);
    free(th);
    return rc;
}
