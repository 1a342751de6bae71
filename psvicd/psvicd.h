/* PSV-ICD (Alg. 2): the paper's multi-core CPU comparison system, SURVEY 8(f)
 * NEXT-4.  A baseline for bench.py's `psv_icd` leg and tests/test_psvicd.py; not the product
 * (csrc/) and not the oracle (oracle/).  See psvicd.c for the algorithm and its readings.
 *
 * Layouts: first/count int32 [ny*nx][V] (first channel and number of non-zero channels of each
 * (voxel, view), count <= K <= 4), vals double [ny*nx][V][K] (A is slice-invariant in parallel
 * beam); y-derived inputs w, e and the image x are float, [nz][V][M] and [nz][ny][nx].  The
 * caller owns every array; psv_create copies what it needs (per-SV tables).
 * Return codes: 0 ok, -1 bad argument (or a band wider than 255 channels), -2 out of memory,
 * -3 no thread could be started. */
#ifndef PSVICD_H
#define PSVICD_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct {
    int nx, ny, nz;
    int nviews, nchannels;
} psv_geom;

/* reading R1: q-GGMRF p, q (= 2), T, sigma; neighbourhood 8 or 26 (R2); positivity (R3) */
typedef struct {
    double p, q, T, sigma;
    int nbhd, positivity;
} psv_prior;

typedef struct {
    int64_t updates, skipped; /* executed / zero-skipped voxel updates of the call */
    double sum_abs_delta;
    double seconds;           /* wall time of the call's iterations */
    int iterations;           /* iterations done by the handle so far */
} psv_stats;

typedef struct psv_handle psv_handle;

/* Alg2:1: tiles each slice into sv_side x sv_side SVs and builds their band tables. */
int psv_create(const psv_geom* g, const psv_prior* pr, int K, const int32_t* first, const int32_t* count,
               const double* vals, int sv_side, psv_handle** out);

/* Alg2:3-20 for n_iters iterations (iteration numbers continue across calls; iterations 1 + k*zero_skip_period run without zero-skip, reading R9).  frac: the share
 * of SVs updated in iterations >= 2 (Alg. 2: 0.2).  x and e (= y - A x for the current x) are
 * updated in place.  nthreads host threads; raster = 1 visits each SV's voxels in raster order
 * instead of a random one (used by the tests).  zero_skip_period as in reading R9. */
int psv_iterate(psv_handle* h, const float* w, float* x, float* e, int n_iters, double frac, uint64_t seed,
                int zero_skip, int zero_skip_period, int nthreads, int raster, psv_stats* st);

void psv_destroy(psv_handle* h);

#ifdef __cplusplus
}
#endif
#endif
