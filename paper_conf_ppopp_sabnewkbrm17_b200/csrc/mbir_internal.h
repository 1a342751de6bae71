// Internal declarations of libmbir (not part of the C-ABI).  See include/mbir.h for the public
// contract and DESIGN.md for the data layout and kernel design.
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

#include <string>
#include <vector>

#include "../../include/mbir.h"

// views per thread of the update kernel when nviews > 128 (VPT = 1 below).  4 is the measured
// best (VPT 2 and 3 were 35-43 % slower); other values are a rebuild
#ifndef MBIR_WIDE_VPT
#define MBIR_WIDE_VPT 4
#endif

namespace mbir {

constexpr int kK = 4;             // max channels per (voxel, view) (reading R5; K=4 for dc > 0.4714 dxy)
constexpr int kMaxNbr = 26;       // 3-D neighbourhood (reading R2)
constexpr int kMaxSvbRows = 64;   // SV-buffer rows: two 32-float windows per band row (pack / write-back)
constexpr int kMaxPhaseSlices = 1024;  // slices of one (z-parity, colour) phase (sched.cu k_flatten)
constexpr int kAutoCapDiv = 12;  // batch_svs = 0: at most N / 12 concurrently updated SVs per slice (R22)
constexpr int kAutoCapMin = 4;

// ---- prior constants, per handle: passed by value in the kernels' parameter blocks ----
struct PriorConst {
    int nnb;                 // 8 or 26
    int dx[kMaxNbr], dy[kMaxNbr], dz[kMaxNbr];
    float b[kMaxNbr];        // b_jr (reading R2)
    float c_phi;             // 1 / (2 sigma^p (T sigma)^(q-p))
    float pq;                // q / p
    float qmp;               // q - p
    float inv_Ts;            // 1 / (T sigma)
    int positivity;
};

// ---- compressed system matrix, per SuperVoxel ----
struct DevA {
    int nsv, S2, V;          // SVs per slice, slots per SV (side^2), views
    int VA;                  // per-voxel record stride (positions) = 32 * view warps * vpt
    int vpt;                 // views per update-kernel thread; records are stored thread-major:
                             // view k sits at position apos(k) so a thread's views are adjacent
    uint32_t* codes;         // [nsv][S2][V] 4 uint8 codes (byte i = channel offset i), quantize_A
    float4* vals;            // [nsv][S2][V] fp32 values, !quantize_A
    uint8_t* off;            // [nsv][S2][V] first channel - band start
    uint8_t* count;          // [nsv][S2][V] channels used (export only)
    float* scale;            // [nsv][S2] amax_j / 255 (quantize_A) or 1
    int32_t* band_start;     // [nsv][V] first channel of the SV band
    uint8_t* band_width;     // [nsv][V] band width (channels)
};

// Record position of view k: thread (warp w, lane l) of the update kernel owns views
// (w*vpt + t)*32 + l, t < vpt, stored at positions (w*32 + l)*vpt + t (one vector load each).
__host__ __device__ __forceinline__ int apos(int k, int vpt)
{
    const int blk = k >> 5;  // = w*vpt + t
    return ((blk / vpt) * 32 + (k & 31)) * vpt + blk % vpt;
}

// byte offsets of the update kernel's shared-memory regions (computed on the host per launch
// configuration and passed in the parameter block, so the kernel addresses them from the
// constant bank instead of recomputing the layout in registers)
struct SmemLayout {
    int sb_e, sb_w, xt, list, flags, tof, red, pri, vscale, vth2, misc, astage, stage_bytes, rscale, rth2, rbs, rbw, cx,
        off_in_stage, mbar, staging, binfo, total;
};

// ---- parameters of the fused SuperVoxel update kernel ----
struct IcdParams {
    int nx, ny, nz_local, z_offset, nz_total;
    int V, M;
    int side, nsvx, nsv, S2;
    int Vs;                  // shared-memory column stride (views), multiple of 32
    int rows;                // shared-memory SVB rows (channels)
    int nvw;                 // view warps (the prior warp is warp nvw)
    DevA A;
    float* e;                // [nz_local][V][M]
    const float* w;          // [nz_local][V][M]
    float* x;                // [nz_local + 2][ny][nx] (halo slice at each end)
    float* theta2;           // [nz_local][nsv][S2]
    float* scratch;          // [max CTAs][Vs][32] e_init tiles of the running SV visits
    float* sv_amount;        // [nz_local][nsv] sum |delta| of the SV's last visit
    const uint8_t* perm;     // [nperm][S2] random permutations of an SV's voxel slots
    int nperm;
    const int* flat;         // phase task list, entries (local slice << 14) | SV
    const int* brange;       // [nbatch + 1]: batch b = flat[brange[b] .. brange[b + 1])
    int* fetch;              // [nbatch] task counters (zeroed per iteration)
    int nbatch;              // batches run by this launch, a grid barrier between two (Alg3:24-27)
    unsigned int* gbar;      // grid-barrier arrival counter of this launch (zeroed per iteration)
    const int* keep;         // optional [list]: 0 = the task's whole tile is zero (zero-skip pre-filter)
    unsigned long long* counters;  // [0] updates [1] skipped [2] sv visits
    double* sum_delta;
    uint64_t seed;
    int iter;
    int zero_skip_active;
    int nwin;         // 32-float windows per band row in the pack / write-back (1, or 2 for > 29 rows)
    int kv;           // voxels per step (1: exact sequential within the SV, 2: voxel pairs)
    int theta2_pass;  // this launch reduces theta2 (Alg1:6) with theta1 and stores it (iteration 1)
    int deterministic;
    unsigned long long* tprof;  // optional [8] phase cycle counters (env MBIR_PHASE_PROFILE)
    PriorConst pc;           // q-GGMRF constants and neighbourhood of this handle (reading R1-R2)
    float* dump;             // optional [dump_cap][4] (voxel bits, theta1, theta2, delta) per update
    unsigned long long* dump_count;
    long long dump_cap;
    SmemLayout lay;          // update-kernel smem layout (filled by launch_svicd)
};

struct SchedParams {
    int nz_local, z_offset;
    int nsvx, nsvy, nsv, nsv_pad;
    int nsel;                // SVs selected per slice this iteration
    int mode;                // 0 all (random order), 1 top by amount, 2 random, 3 all in index order
    int max_group;
    uint64_t seed;
    int iter;
    const float* sv_amount;
    int* task_list;
    int* task_count;
};

// kernels / launchers (sysmatrix.cu, icd.cu, sched.cu, aux.cu)
cudaError_t build_sysmatrix(const mbir_geometry& g, const double* d_angles_cs, int side, int nsvx,
                            int nsvy, bool quantize, DevA& A, int* d_err, int* d_maxoff,
                            cudaStream_t st);
// the fused update kernel (svicd_impl.cuh, instantiated in svicd_n*_*.cu): per CTA nvw / cl view warps + the delta warp + the prior
// warp, vpt = 4 (or 1 for <= 128 views) views per lane; cl = 2: a 2-CTA cluster splits a task's views
int svicd_smem_bytes(const IcdParams& p, int vpt, int nnb, bool quantize, int cl);
int svicd_resident_ctas(const IcdParams& p, int vpt, int nnb, bool quantize, int cl);
int svicd_scratch_floats(int vpt, int nwin);  // per-CTA e_init scratch tile
cudaError_t launch_svicd(const IcdParams& p, int vpt, int nnb, bool quantize, int cl, int grid, cudaStream_t st);
cudaError_t launch_theta2(const IcdParams& p, bool quantize, cudaStream_t st);
cudaError_t launch_forward(const IcdParams& p, bool quantize, const float* y, cudaStream_t st);
cudaError_t launch_probe(const IcdParams& p, bool quantize, int nnb, const int64_t* vox, int n,
                         float* out3, cudaStream_t st);
cudaError_t launch_select(const SchedParams& sp, cudaStream_t st);
// Build the flat, slice-interleaved task list of each (z-parity, colour) phase and its batch
// ranges (Alg3:24-27): flat[ph][...], brange[ph][b] (b = 0..nb), ph = parity*4 + colour.
cudaError_t launch_flatten(const int* task_list, const int* task_count, int nz_local, int z_offset,
                           int parities, int max_group, int batch, int thr, int nb, int* flat,
                           int* brange, cudaStream_t st);
// FBP initial image (fbp.cu): q = ramp-filtered y (scratch [nz][V][M]), x = clip(backprojection)
cudaError_t launch_fbp(const mbir_geometry& g, const double* d_cs, const float* y, float* q, float* x,
                       int positivity, cudaStream_t st);
// zero-skip pre-filter of a phase list (sched.cu): keep[t] = 0 iff task t's whole tile is zero
cudaError_t launch_zero_flags(const int* flat, const int* brange, const float* x, int nx, int ny,
                              int nz_local, int z_offset, int nz_total, int side, int nsvx, int nnb,
                              int max_tasks, int* keep, cudaStream_t st);
cudaError_t launch_rmse_partial(const float* x, const float* g, int64_t n, double* acc,
                                cudaStream_t st);
cudaError_t launch_check_finite(const float* a, int64_t n, int nonneg, int* flag, cudaStream_t st);
cudaError_t launch_export_sysmatrix(const DevA& A, int nx, int ny, int side, int nsvx,
                                    const int64_t* vox, int nvox, int32_t* first, int32_t* count,
                                    float* vals, uint8_t* codes, float* scales,
                                    const mbir_geometry& g, const double* d_angles_cs,
                                    cudaStream_t st);

}  // namespace mbir
