/*
 * oracle.h -- plain, slow, sequential CPU oracle for the GPU-ICD hot path.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load this library.  The product
 * (paper_conf_ppopp_sabnewkbrm17_b200/, libmbir.so) never links, imports or calls it,
 * and it shares no code, header, table or constant generator with the CUDA path.
 *
 * What it computes (PAPER.md = /root/reference/PAPER.md, "P:n" = line n):
 *   - Alg. 1 ("Updating Single Voxel"): theta1 = -sum w*A*e, theta2 = sum w*A^2,
 *     delta = func(v, theta1, theta2, neighbours), v += delta, e -= A*delta.
 *   - "traditional" sequential ICD over all voxels in random order,
 *     with zero-skipping.
 *   - The system matrix A of a parallel-beam scanner as
 *     area(strip_i ∩ pixel_j)/dchannel, by explicit polygon clipping (reading R4).
 *   - The uint8 quantisation of A (reading R6).
 *   - The q-GGMRF prior and its symmetric-bound surrogate that realise `func`
 *     (P:107-109 leaves func undefined; readings R1-R3).
 *   - The MAP cost f(x) = 1/2 (y-Ax)^T W (y-Ax) + sum_{pairs} b_jr rho(x_j - x_r)
 *     (Eq. 1 at P:351, with the 1/2 implied by Alg. 1's thetas; reading R7).
 *
 * All arithmetic is IEEE double, single thread (orc_icd_run_zpar: one thread per slice of a
 * z-parity on POSIX threads, an exact serialisation), no blocking/fusion/reordering beyond the definitions above.  Pins (tests/test_oracle_pins.py) tie it to closed forms,
 * brute force, paper-printed values and invariants.
 *
 * Parity status per function:
 *   orc_strip_pixel_area / orc_sysmatrix_*  pinned (P1 brute force, P2 worked entries + area invariant)
 *   orc_quantize_column                     pinned (P11 codec special values)
 *   orc_rho / orc_phi                        pinned (P8 finite differences, limit, majorisation)
 *   orc_voxel_update / orc_icd_run           pinned (P3 closed form, P4 monotone cost, P5 e-consistency,
 *                                            P6 dense solve, P7 Gauss-Seidel equivalence)
 *   orc_cost                                 pinned (P4, P6 via independent numpy evaluation)
 */
#ifndef MBIR_ORACLE_H
#define MBIR_ORACLE_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* Parallel-beam geometry (reading R4).  Image [nz][ny][nx] (x fastest),
 * pixel pitch dxy (mm), slice pitch = dxy.  Views theta_k = k*pi/nviews over [0, pi)
 * unless `angles` is given.  Channel i covers [t0 + i*dc, t0 + (i+1)*dc) with
 * t0 = -nchannels*dc/2 + center_offset*dc. */
typedef struct {
    int nx, ny, nz;
    double dxy;
    int nviews, nchannels;
    double dchannel;
    double center_offset;
    const double* angles; /* NULL -> k*pi/nviews */
} orc_geom;

/* q-GGMRF prior (reading R1): rho(D) = |D|^p/(p s^p) * u/(1+u), u = |D/(T s)|^(q-p).
 * nbhd = 8 (2-D, in-slice) or 26 (3-D).  positivity: clip the update at 0 (reading R3). */
typedef struct {
    double p, q, T, sigma;
    int nbhd;
    int positivity;
} orc_prior;

typedef struct {
    int64_t updates;   /* executed (non-skipped) voxel updates (P:277 equit accounting) */
    int64_t skipped;   /* zero-skipped visits */
    double sum_abs_delta;
} orc_stats;

/* ---- system matrix (reading R4/R5) ---- */

/* Exact area of {pixel square centred (cx,cy), side d} ∩ {tlo <= x*cos + y*sin <= thi},
 * by Sutherland-Hodgman clipping of the square against the two half-planes + shoelace. */
double orc_strip_pixel_area(double cx, double cy, double d, double c, double s,
                            double tlo, double thi);

/* View angle k (reading R4). */
double orc_view_angle(const orc_geom* g, int k);

/* Column of A for in-slice voxel (ix, iy): for each view k, first[k] = first channel,
 * count[k] = number of channels (0..K), vals[k*K + i] = A_{first+i, j} (unused slots 0).
 * Returns the maximum count seen (caller checks <= K). */
int orc_sysmatrix_column(const orc_geom* g, int ix, int iy, int K,
                         int32_t* first, int32_t* count, double* vals);

/* Whole slice-plane A (A is slice-invariant in parallel beam): voxel j = iy*nx + ix,
 * arrays first/count [nx*ny][nviews], vals [nx*ny][nviews][K].  Returns max count. */
int orc_sysmatrix_build(const orc_geom* g, int K, int32_t* first, int32_t* count, double* vals);

/* uint8 codec of P:267-269 (reading R6): amax = max_i A_ij over the voxel's entries,
 * code = (uint8) floor(A/amax*255 + 0.5).  codes laid out like vals.  Returns amax. */
double orc_quantize_column(const double* vals, const int32_t* count, int nviews, int K,
                           uint8_t* codes);

/* ---- prior (reading R1-R2) ---- */
double orc_rho(double delta, const orc_prior* pr);
/* phi(D) = rho'(D) / (2 D), with its limit at D = 0 (requires q = 2 there). */
double orc_phi(double delta, const orc_prior* pr);
/* Neighbour weight b_jr for offset (dx,dy,dz): 1/distance normalised so an interior
 * voxel's weights sum to 1 (reading R2).  0 for (0,0,0) or offsets outside the nbhd. */
double orc_nbr_weight(int dx, int dy, int dz, int nbhd);

/* ---- Alg. 1 ---- */
/* Computes theta1, theta2 and delta for voxel j = (iz*ny+iy)*nx+ix at the current
 * (x, e).  If apply != 0: x_j += delta and e -= A_j*delta (Alg1:8-11).
 * col_* is the voxel's in-slice column (from orc_sysmatrix_*). */
void orc_voxel_update(const orc_geom* g, const orc_prior* pr, int K,
                      const int32_t* col_first, const int32_t* col_count, const double* col_vals,
                      const double* w, double* x, double* e, int64_t j, int apply,
                      double* theta1, double* theta2, double* delta);

/* Sequential ICD.  For each of n_equits sweeps: visit all nz*ny*nx voxels,
 * in `order` (if non-NULL, `order_len` voxel indices per sweep) or a fresh random
 * permutation (splitmix64 Fisher-Yates seeded from (seed, sweep number)).  Zero-skip
 * (reading R9): when zero_skip != 0 and the 1-based sweep number (first_sweep + s) > 1,
 * skip voxel j iff x_j and all its neighbours are exactly 0 -- except in sweeps whose number
 * is a multiple of zero_skip_period (> 0), which re-examine every voxel.
 * e must equal y - A x on entry (use orc_error_sinogram).  If dump != NULL it receives
 * (j, theta1, theta2, delta) for every executed update, in order (dump_cap entries max).
 * Returns number of dump entries written. */
int64_t orc_icd_run(const orc_geom* g, const orc_prior* pr, int K,
                    const int32_t* first, const int32_t* count, const double* vals,
                    const double* w, double* x, double* e,
                    int n_equits, int first_sweep, uint64_t seed, int zero_skip, int zero_skip_period,
                    const int64_t* order, int64_t order_len,
                    double* dump, int64_t dump_cap, orc_stats* st);

/* The same ICD with slices of one z-parity run concurrently on nthreads POSIX threads:
 * per sweep, parity 0 slices then parity 1 slices, each slice in its own random order.  An
 * exact serialisation of sequential ICD (same-parity slices share no data; see oracle.c).
 * Returns 0, or -1 on allocation failure.  Stats are accumulated into *st. */
int orc_icd_run_zpar(const orc_geom* g, const orc_prior* pr, int K, const int32_t* first,
                     const int32_t* count, const double* vals, const double* w, double* x,
                     double* e, int n_equits, int first_sweep, uint64_t seed, int zero_skip,
                     int zero_skip_period, int nthreads, orc_stats* st);

/* e = y - A x for the whole volume (per slice, same A). */
void orc_error_sinogram(const orc_geom* g, int K, const int32_t* first, const int32_t* count,
                        const double* vals, const double* y, const double* x, double* e);

/* f(x) = 1/2 sum w e^2 + sum_{unordered neighbour pairs} b_jr rho(x_j - x_r), e = y - A x. */
double orc_cost(const orc_geom* g, const orc_prior* pr, int K, const int32_t* first,
                const int32_t* count, const double* vals, const double* y, const double* w,
                const double* x);

/* RMSE in Hounsfield units (reading R12): 1000*sqrt(mean((a-b)^2))/mu_water. */
double orc_rmse_hu(const double* a, const double* b, int64_t n, double mu_water);

#ifdef __cplusplus
}
#endif
#endif
