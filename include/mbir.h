/*
 * mbir.h -- C-ABI of libmbir: a B200-native (sm_100a) implementation of the GPU-ICD hot path
 * of Sabne et al., "Model-based Iterative CT Image Reconstruction on GPUs", PPoPP'17.
 *
 * Citations: "P:n" = line n of the paper text; "Alg k:i" = line i
 * of Algorithm k.  DESIGN.md lists every reading of a passage the paper leaves open (R1...).
 *
 * What the library computes: model-based iterative reconstruction by SuperVoxel ICD.
 *   minimise  f(x) = 1/2 (y - A x)^T W (y - A x) + sum_{j~r} b_jr rho(x_j - x_r),  x >= 0
 * (Eq. 1 at P:351 plus the prior of reading R1) by Alg. 1 single-voxel updates
 * run with the three levels of parallelism of P:155-161: within a voxel (threads over the
 * voxel's views), within a SuperVoxel (sequential-exact, pipelined across warps), and across
 * SuperVoxels of one checkerboard colour and across slices.
 *
 * Conventions shared by every call:
 *   - All functions are extern "C", never throw, and return 0 (MBIR_OK) or a negative code.
 *     mbir_last_error(h) gives a human-readable message for the last failure on h.
 *   - Image layout [nz_local][ny][nx] float32, x fastest, units mm^-1.
 *   - Sinogram layout [nz_local][nviews][nchannels] float32, channel fastest (one sinogram
 *     column per view angle).
 *   - `where` = MBIR_HOST (pageable or pinned host memory) or MBIR_DEVICE (a device pointer on
 *     the handle's device, e.g. a torch CUDA tensor's data_ptr()).  All calls COPY; the caller
 *     keeps ownership of every buffer it passes.  Device-side work is ordered on the handle's
 *     stream; calls return after that stream has been synchronised unless stated otherwise.
 *   - The library owns all of its device memory (allocated in mbir_create / set_sinogram and
 *     released by mbir_destroy).
 */
#ifndef MBIR_H
#define MBIR_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define MBIR_OK 0
#define MBIR_EINVAL (-1)   /* bad argument / unsupported size */
#define MBIR_ENOMEM (-2)   /* device or host allocation failed */
#define MBIR_ECUDA (-3)    /* CUDA runtime error (message in mbir_last_error) */
#define MBIR_ESTATE (-4)   /* call out of order (e.g. reconstruct before set_sinogram) */
#define MBIR_ENUMERIC (-5) /* NaN/Inf detected in the state */
#define MBIR_ENCCL (-6)    /* NCCL error (multi-GPU) */
#define MBIR_ENOTSUP (-7)  /* feature not built in */

#define MBIR_HOST 0
#define MBIR_DEVICE 1

typedef struct mbir_handle mbir_handle;

/* Parallel-beam scanner + image grid (readings R4, R5).
 * Pixel centres ((ix-(nx-1)/2)*dxy, (iy-(ny-1)/2)*dxy); slices have pitch dxy.
 * View k has angle angles[k] (host array of nviews doubles, copied) or k*pi/nviews if NULL.
 * Channel i covers [t0 + i*dchannel, t0 + (i+1)*dchannel), t0 = -nchannels*dchannel/2 +
 * center_offset*dchannel.  nz_local slices starting at global slice z_offset of nz_total
 * (z-slab partition across ranks). */
typedef struct mbir_geometry {
    int nx, ny;
    int nz_local, z_offset, nz_total;
    double dxy;
    int nviews, nchannels;
    double dchannel;
    double center_offset;
    const double* angles;
} mbir_geometry;

/* q-GGMRF prior (reading R1): rho(D) = |D|^p/(p sigma^p) * u/(1+u), u = |D/(T sigma)|^(q-p).
 * Requirements: 1 <= p <= 2, q == 2, T > 0, sigma > 0.  neighborhood = 8 (in-slice) or 26
 * (3-D, slices of pitch dxy); weights b_jr ~ 1/distance summing to 1 (reading R2), free boundary.
 * positivity != 0 clips every update at 0 (reading R3). */
typedef struct mbir_prior {
    double p, q, T, sigma;
    int neighborhood;
    int positivity;
} mbir_prior;

/* Algorithmic options (Table 1).  Zero-initialise and
 * call mbir_default_options() for the defaults. */
typedef struct mbir_options {
    int sv_side;           /* SuperVoxel side s; tiles of s x s voxels, default 9   */
    double sv_fraction;    /* fraction of SVs per iteration >= 2, default 0.25  */
    int batch_svs;         /* BATCH_SIZE: SVs per slice per launch (Alg3:25); 0 = auto: a whole
                              checkerboard colour group per launch when the phase spans enough
                              slices that at most cap = max(4, N / 12) SVs of one slice (N =
                              max(nx, ny)) run at once, else batches of cap SVs per slice (no
                              threshold); default 0 (reading R22)                       */
    int batch_threshold;   /* Alg3:26-27: drop a group's remainder smaller than this; -1 =
                              batch_svs/4; ignored when batch_svs == 0                   */
    int zero_skip;         /* P:115, default 1 (never in iteration 1; reading R9)               */
    int quantize_A;        /* 1: A as uint8 codes + per-voxel scale, 0: fp32 values */
    uint64_t seed;         /* voxel-order / random-SV-selection seed                            */
    int deterministic;     /* debug: every iteration visits all SVs one at a time (one CTA) in
                              the order z-parity half (3-D prior only), colour, SV rank within
                              the colour (SV index order), slice; voxels in raster order        */
    int cluster;           /* CTAs per SV task in the update kernel: 0 = auto (1, or 2 when one
                              CTA's shared memory cannot hold the SV buffer: large SVs, e.g.
                              side 11-15 at the paper's 720 x 1024 geometry), 1 = one CTA owns a
                              task, 2 = a 2-CTA thread-block cluster splits the task's views
                              (each holds half the SV buffer; one partial sum per voxel crosses
                              distributed shared memory; two SMs per SV).  2 needs > 128 views;
                              an odd number of 128-view warps is padded by one warp of empty
                              views (zero records).  Same arithmetic either way.  SV
                              bands of up to 61 rows (channels) per view are supported          */
    int zero_skip_period;  /* with zero_skip: iterations 1 + k*zero_skip_period, k >= 1 (numbers
                              counted from the last set_sinogram / set_image) run
                              WITHOUT zero-skipping on a random sv_fraction of the SVs, so voxels
                              frozen at 0 are re-examined and the fixed point stays the MAP
                              estimate; 0 = the plain heuristic of P:115, whose fixed point can
                              differ from the MAP (reading R9).  Default 4                      */
    int voxels_per_step;   /* voxels of one SV updated concurrently by the update kernel (the
                              paper's intra-SV parallelism): 1 = exact sequential
                              ICD inside the SV (one voxel per step); 2 = voxel pairs: both
                              voxels' theta1, theta2 and prior terms from the same e and x (the
                              second does not see the first's update), then both applied; needs
                              uint8 A and one CTA per task (else EINVAL).  0 = auto = 1 (pairs
                              measured 5 % slower on the bench workload) */
} mbir_options;

/* Placement and (optional) multi-GPU slab partition.  device: CUDA ordinal.  stream: a
 * cudaStream_t on which every call orders its device work (NULL = the library creates its own
 * blocking stream, implicitly ordered with the legacy default stream).  Device buffers passed
 * to any call must be complete with respect to that stream (pass the stream that produced
 * them; the Python binding passes torch's current stream).  For nranks > 1, nccl_unique_id points to
 * the 128-byte ncclUniqueId produced by mbir_nccl_unique_id() on rank 0 and broadcast by the
 * caller (e.g. over a torch.distributed process group); rank r must own slices
 * [z_offset, z_offset + nz_local) with slabs contiguous in rank order. */
typedef struct mbir_dist {
    int device;
    void* stream;
    int rank, nranks;
    const void* nccl_unique_id;
} mbir_dist;

/* Per-call statistics (P:277 equit accounting; Table 1). */
typedef struct mbir_stats {
    int64_t updates;       /* executed (non-skipped) voxel updates, all ranks        */
    int64_t skipped;       /* zero-skipped voxel visits                               */
    int64_t sv_visits;     /* (SV, slice) tasks executed                              */
    int64_t iterations;    /* outer iterations (Alg3:16) executed by this call       */
    double equits;         /* updates / (nx*ny*nz_total)                              */
    double seconds;        /* device time of this call (CUDA events)                  */
    double sum_abs_delta;  /* sum |delta| over the executed updates                   */
    int64_t launches;      /* kernel launches issued by this call                     */
    double kernel_seconds; /* summed device time of the fused update-kernel launches,
                              CUDA events on the handle's stream around each launch     */
    int64_t kernel_launches; /* fused update-kernel launches                           */
    int64_t sv_visits_empty; /* of sv_visits: tasks whose every voxel was zero-skipped (no
                                SV-buffer traffic; reading R9)                           */
} mbir_stats;

/* Sizes of the internal layout (for tests, benchmarks and buffer allocation). */
typedef struct mbir_sizes {
    int nsv_x, nsv_y, nsv;          /* SuperVoxel tiles per slice                         */
    int K;                          /* max channels per (voxel, view): 4                  */
    int band_max;                   /* max SV band width over (SV, view), channels        */
    int svb_rows;                   /* rows of the shared-memory SV buffer (>= band_max)  */
    int threads_per_cta;            /* update-kernel block size                            */
    int cluster;                    /* update-kernel CTAs per SV task (1 or 2)             */
    int resident_ctas;              /* update-kernel CTAs resident at once (occupancy)     */
    int smem_bytes;                 /* update-kernel dynamic shared memory                 */
    int64_t nnz;                    /* total non-zeros of the slice-plane system matrix    */
    int64_t a_bytes;                /* device bytes of the compressed A                   */
    int64_t band_entries;           /* sum over (SV, view) of band widths                  */
    int max_group;                  /* SVs of one checkerboard colour per slice (max)     */
    int voxels_per_step;            /* update-kernel voxels per SV step in effect (1, 2)  */
} mbir_sizes;

/* Fill defaults: sv_side 9, sv_fraction 0.25, batch_svs 0, batch_threshold -1, zero_skip 1,
 * quantize_A 1, seed 3000, deterministic 0, cluster 0 (auto), zero_skip_period 4,
 * voxels_per_step 0 (auto). */
void mbir_default_options(mbir_options* o);
/* p 1.2, q 2, T 1, sigma 0.005, neighborhood 26, positivity 1. */
void mbir_default_prior(mbir_prior* p);

/* Build a reconstruction context: validates arguments (MBIR_EINVAL), computes the system
 * matrix on the device in double precision (strip-area model, reading R4) and compresses it
 * per SuperVoxel (per-view band offsets + uint8 codes or fp32 values),
 * builds the SV tiling and scheduler state, and (nranks > 1) joins the NCCL communicator.
 * *out is set only on success.  Errors: EINVAL, ENOMEM, ECUDA, ENCCL. */
int mbir_create(const mbir_geometry* g, const mbir_prior* p, const mbir_options* o,
                const mbir_dist* d, mbir_handle** out);

/* Load the measured sinogram y and its weights w (inverse noise variance), both
 * [nz_local][nviews][nchannels].  Resets the error sinogram e = y - A x for the current image
 * (Alg. 1 input) and the scheduler state.  theta2 = A^T W A (Alg1:6), which depends only on w,
 * is computed by the next iteration's update kernel (the first iteration visits every voxel),
 * or by a separate pass first when a batch threshold could drop tasks.  Errors: EINVAL (NULL,
 * NaN/Inf or negative w), ECUDA. */
int mbir_set_sinogram(mbir_handle* h, const float* y, const float* w, int where);

/* Set the image (warm start / resume; default 0).  x0 == NULL sets 0.  Recomputes e = y - A x
 * if a sinogram is loaded.  Errors: EINVAL (negative values with positivity), ECUDA. */
int mbir_set_image(mbir_handle* h, const float* x0, int where);

/* Set the image to the filtered back-projection of the loaded sinogram y (Ram-Lak filter by
 * direct convolution, linearly interpolated back-projection, clipped at 0 with positivity;
 * Kak & Slaney ch. 3) and recompute e = y - A x.  An initial image only: the paper does not
 * state one (reading R23) and ICD converges to the same MAP point from any start.
 * Collective across ranks (halo exchange).  Uses a temporary [nz_local][nviews][nchannels]
 * device buffer.  Errors: ESTATE (no sinogram), ENOMEM, ECUDA, ENCCL. */
int mbir_init_fbp(mbir_handle* h);

/* Run whole iterations of GPU-ICD (Alg. 3 lines 16-31) until at least `equits` equits of
 * executed updates have been done by this call (one equit = nx*ny*nz_total updates).
 * Collective across ranks.  st may be NULL.  Errors: ESTATE (no sinogram), ENUMERIC, ECUDA,
 * ENCCL. */
int mbir_reconstruct(mbir_handle* h, double equits, mbir_stats* st);

/* Run exactly n_iterations iterations (for convergence curves).  Same errors. */
int mbir_iterate(mbir_handle* h, int n_iterations, mbir_stats* st);

/* Copy the current image [nz_local][ny][nx] into x.  Errors: EINVAL, ECUDA. */
int mbir_get_image(mbir_handle* h, float* x, int where);

/* Copy the current error sinogram e [nz_local][nviews][nchannels] (test hook). */
int mbir_get_error_sinogram(mbir_handle* h, float* e, int where);

/* RMSE in Hounsfield units of the current image against `golden` ([nz_local][ny][nx],
 * device or host), 1000*sqrt(mean((x-g)^2))/mu_water (reading R12), reduced over all
 * ranks.  Device reduction. */
int mbir_rmse_hu(mbir_handle* h, const float* golden, int where, double mu_water, double* out);

int mbir_query_sizes(const mbir_handle* h, mbir_sizes* s);

/* Export the slice-plane system matrix in the plain layout (test hook, host buffers, each may
 * be NULL): first/count int32 [ny*nx][nviews] (first channel, number of channels), values
 * float32 [ny*nx][nviews][K] (fp32 of the double-precision strip areas / dchannel; unused
 * slots 0), codes uint8 [ny*nx][nviews][K] (P:267 codec), scales float32 [ny*nx]
 * (max_j(A)/255). */
int mbir_get_sysmatrix(mbir_handle* h, int32_t* first, int32_t* count, float* values,
                       uint8_t* codes, float* scales);

/* Same for n selected in-slice voxels (flat iy*nx + ix): row i of each output describes
 * voxels[i] (test hook for full-size geometries). */
int mbir_get_sysmatrix_columns(mbir_handle* h, const int64_t* voxels, int n, int32_t* first,
                               int32_t* count, float* values, uint8_t* codes, float* scales);

/* Alg. 1 steps 1-7 for n voxels at the CURRENT state, without applying them (test hook):
 * voxels are flat local indices (z*ny + y)*nx + x; theta1/theta2/delta are host arrays of n
 * floats, computed on the device from the library's A representation, e, w and x. */
int mbir_probe_update(mbir_handle* h, const int64_t* voxels, int n, float* theta1,
                      float* theta2, float* delta);

/* Test hook (the z-slab partition of DESIGN.md section 9 without several GPUs): link n handles
 * created on ONE device with nranks = n, rank = i, no NCCL id, owning consecutive slabs of one
 * volume (rank order), so that their halo exchanges (mbir_halo_plan) become device-to-device
 * copies between the handles behind a host barrier.  The caller must then drive all of them
 * concurrently (one host thread per handle) with the same sequence of collective calls
 * (set_image, init_fbp, iterate, reconstruct).  Counters and RMSE are NOT reduced across linked
 * handles (each reports its own slab).  Errors: EINVAL (wrong ranks/order/device, already
 * linked), ENOMEM. */
int mbir_link_slabs(mbir_handle** handles, int n);

/* Test hook: record every voxel update the fused update kernel executes from now on -- the
 * (theta1, theta2, delta) of Alg. 1 steps 3-8 exactly as the kernel's delta chain
 * used them.  capacity = entries kept (0 = off; frees the buffer).  With voxel pairs
 * (voxels_per_step 2) both updates of a pair are computed from the same state: the second is
 * recorded right after the first with MBIR_DUMP_SAME_STATE set in its voxel index.  In
 * deterministic mode (one CTA) the record is the exact update sequence.  Errors: EINVAL,
 * ENOMEM. */
int mbir_set_update_dump(mbir_handle* h, int64_t capacity);

#define MBIR_DUMP_SAME_STATE ((int64_t)1 << 62) /* update record flag (mbir_set_update_dump) */

/* Copy up to cap recorded updates into host arrays (voxels: local flat (z*ny + y)*nx + x,
 * | MBIR_DUMP_SAME_STATE for the second update of a pair;
 * theta1, theta2, delta float32), set *n to the number recorded since the last call (which
 * can exceed cap and the capacity: then the record was truncated), and restart the record.
 * Errors: EINVAL, ESTATE (no dump buffer), ECUDA. */
int mbir_get_update_dump(mbir_handle* h, int64_t cap, int64_t* voxels, float* theta1,
                         float* theta2, float* delta, int64_t* n);

/* Test hook (scheduler, P:203-225 / Alg3:17-23): copy the SV selection of the most recent
 * iteration and the update amounts (host buffers, each may be NULL).  task_list int32
 * [nz_local][4 colours][max_group] (SV indices of the colour group in selection order; entries
 * past task_count are stale), task_count int32 [nz_local][4], amount float32 [nz_local][nsv]
 * (sum |delta| of each SV's most recent visit, the key of the next "top" selection). */
int mbir_get_schedule(mbir_handle* h, int32_t* task_list, int32_t* task_count, float* amount);

/* Multi-GPU bootstrap: write a fresh 128-byte ncclUniqueId into id (call on rank 0 only).
 * Returns ENOTSUP if libnccl.so.2 cannot be loaded. */
int mbir_nccl_unique_id(void* id128);

/* z-slab halo schedule (host-only, no GPU).  After the half-iteration
 * that updated the slices of global parity `parity` (0 or 1; -1 = both boundary slices, as after
 * mbir_set_image), rank `rank` of `nranks` owning global slices [z_offset, z_offset + nz_local)
 * exchanges boundary slices with its neighbours.  Writes up to 4 operations to ops (int32[4][3]:
 * peer rank, 1 = send / 0 = receive, local storage slice where 0 is the lower halo, 1..nz_local
 * the owned slices and nz_local + 1 the upper halo) in the order they are posted inside one NCCL
 * group, and returns how many (>= 0), or MBIR_EINVAL.  mbir_reconstruct uses exactly this plan. */
int mbir_halo_plan(int z_offset, int nz_local, int rank, int nranks, int parity, int32_t* ops);

void mbir_destroy(mbir_handle* h);
const char* mbir_strerror(int code);
const char* mbir_last_error(const mbir_handle* h);

#ifdef __cplusplus
}
#endif
#endif /* MBIR_H */
