// Device-side SuperVoxel scheduler and small reduction kernels.
//
// Paper, Alg. 3 lines 17-23: iteration 1 updates all SVs; even iterations the
// top 25 % by "update amount"; odd iterations a random 25 % (P:225 raises PSV-ICD's 20 % to 25 %
// for GPU load balance); the chosen set is split into 4 checkerboard groups whose members share
// no boundary (Fig. 3).  Reading R14: the update amount is sum |delta| of the SV's
// most recent visit, the selection is made per slice, ties go to the lower SV index, and the
// random subset (and iteration 1's random order) is uniform without replacement from a
// counter-based hash of (seed, iteration, SV) -- the same for every slice, so the flat task list
// (rank r of every slice, then r + 1, ...) runs one SV at all slices of a phase back to back and
// the concurrently running CTAs share that SV's A records through L2 (A is slice-invariant in
// parallel beam, cross-slice A reuse).
//
// One CTA per slice: keys in shared memory -> bitonic sort -> the first nsel keys are the
// selection, in key order -> a block-wide scan of 4 packed 16-bit colour counters places every
// selected SV into its colour's task list (order preserved).
#include "mbir_internal.h"

namespace mbir {

namespace {

__device__ __forceinline__ uint64_t mix64s(uint64_t z)
{
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
    return z ^ (z >> 31);
}

constexpr int kSelThreads = 1024;

__global__ void __launch_bounds__(kSelThreads) k_select(const SchedParams S)
{
    extern __shared__ unsigned long long keys[];  // [nsv_pad]
    __shared__ unsigned long long wscan[kSelThreads / 32];
    const int z = blockIdx.x;
    const int n = S.nsv_pad;
    for (int i = threadIdx.x; i < n; i += blockDim.x) {
        unsigned long long key = ~0ull;
        if (i < S.nsv) {
            if (S.mode == 1) {
                const float a = S.sv_amount[(size_t)z * S.nsv + i];
                const uint32_t bits = __float_as_uint(fmaxf(a, 0.f));
                key = ((unsigned long long)(~bits) << 32) | (unsigned)i;  // larger amount first
            } else if (S.mode == 3) {
                key = (unsigned long long)i;
            } else {
                const uint64_t h = mix64s(S.seed ^ 0x5bd1e995ULL ^ mix64s(((uint64_t)S.iter << 40) ^ (uint64_t)i));
                key = ((unsigned long long)(uint32_t)(h >> 32) << 32) | (unsigned)i;
            }
        }
        keys[i] = key;
    }
    __syncthreads();
    if (S.mode != 3) {
        for (int k = 2; k <= n; k <<= 1)
            for (int j = k >> 1; j > 0; j >>= 1) {
                for (int i = threadIdx.x; i < n; i += blockDim.x) {
                    const int ixj = i ^ j;
                    if (ixj > i) {
                        const bool up = (i & k) == 0;
                        const unsigned long long a = keys[i], b = keys[ixj];
                        if ((a > b) == up) {
                            keys[i] = b;
                            keys[ixj] = a;
                        }
                    }
                }
                __syncthreads();
            }
    }
    // colour of each selected SV, 4 x 16-bit counters packed in a uint64
    const int nsel = S.nsel;
    const int per = (nsel + blockDim.x - 1) / blockDim.x;
    const int b0 = threadIdx.x * per, b1 = min(nsel, b0 + per);
    unsigned long long local = 0;
    for (int q = b0; q < b1; ++q) {
        const int s = (int)(keys[q] & 0xffffffffu);
        const int col = ((s % S.nsvx) & 1) + 2 * ((s / S.nsvx) & 1);
        local += 1ull << (16 * col);
    }
    // block exclusive scan of `local`
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    unsigned long long incl = local;
    for (int o = 1; o < 32; o <<= 1) {
        const unsigned long long t = __shfl_up_sync(0xffffffffu, incl, o);
        if (lane >= o) incl += t;
    }
    if (lane == 31) wscan[wid] = incl;
    __syncthreads();
    if (wid == 0) {
        unsigned long long v = lane < (int)(blockDim.x >> 5) ? wscan[lane] : 0ull;
        for (int o = 1; o < 32; o <<= 1) {
            const unsigned long long t = __shfl_up_sync(0xffffffffu, v, o);
            if (lane >= o) v += t;
        }
        wscan[lane] = v;  // inclusive over warps
    }
    __syncthreads();
    unsigned long long excl = incl - local + (wid > 0 ? wscan[wid - 1] : 0ull);
    const unsigned long long total = wscan[(blockDim.x >> 5) - 1];
    for (int q = b0; q < b1; ++q) {
        const int s = (int)(keys[q] & 0xffffffffu);
        const int col = ((s % S.nsvx) & 1) + 2 * ((s / S.nsvx) & 1);
        const int p = (int)((excl >> (16 * col)) & 0xffffu);
        S.task_list[((size_t)z * 4 + col) * S.max_group + p] = s;
        excl += 1ull << (16 * col);
    }
    if (threadIdx.x < 4) S.task_count[z * 4 + threadIdx.x] = (int)((total >> (16 * threadIdx.x)) & 0xffffu);
}

// One block per phase ph = parity*4 + colour (Alg3:23-27).  Slices of that z-parity contribute
// their colour group; a slice's group is cut into batches of B and, with a threshold, the
// batches from the first one with fewer than thr SVs left are dropped ("break", reading R15).
// Kept tasks are interleaved round-robin over slices (rank r of every slice, then r+1, ...),
// so each batch is a contiguous range and concurrent CTAs work on different slices.
// (mbir_create rejects volumes with more than kMaxPhaseSlices slices in one phase)
__global__ void k_flatten(const int* __restrict__ task_list, const int* __restrict__ task_count,
                          int nz_local, int z_offset, int parities, int max_group, int B, int thr,
                          int nb, int* __restrict__ flat, int* __restrict__ brange)
{
    __shared__ int zl[kMaxPhaseSlices], K[kMaxPhaseSlices];
    __shared__ int s_n, s_maxK;
    const int ph = blockIdx.x, parity = ph / 4, colour = ph % 4;
    if (threadIdx.x == 0) {
        int n = 0, mk = 0;
        for (int z = 0; z < nz_local && n < kMaxPhaseSlices; ++z) {
            if (parities == 2 && ((z_offset + z) & 1) != parity) continue;
            const int cnt = task_count[z * 4 + colour];
            int k = cnt;
            if (thr > 0) {
                k = 0;
                for (int b = 0; b * B < cnt; ++b) {
                    if (cnt - b * B < thr) break;
                    k = min(cnt, (b + 1) * B);
                }
            }
            zl[n] = z;
            K[n] = k;
            mk = max(mk, k);
            ++n;
        }
        s_n = n;
        s_maxK = mk;
    }
    __syncthreads();
    const int n = s_n, maxK = s_maxK;
    const size_t cap = (size_t)nz_local * max_group;
    for (int e = threadIdx.x; e < n * maxK; e += blockDim.x) {
        const int zi = e % n, r = e / n;
        if (r >= K[zi]) continue;
        int pos = 0;
        for (int j = 0; j < n; ++j) pos += min(K[j], r) + ((j < zi && K[j] > r) ? 1 : 0);
        const int z = zl[zi];
        flat[ph * cap + pos] = (z << 14) | task_list[((size_t)z * 4 + colour) * max_group + r];
    }
    for (int b = threadIdx.x; b <= nb; b += blockDim.x) {
        int s = 0;
        for (int j = 0; j < n; ++j) s += min(K[j], b * B);
        brange[ph * (nb + 1) + b] = s;
    }
}

// Zero-skip pre-filter of one phase's task list (iterations >= 2, no batching).  An SV visit is
// fully skipped (reading R9) iff every in-volume x of its tile -- the SV, its 1-voxel ring
// and, with the 26-neighbourhood, the slices z +- 1 -- is 0.  During a phase only SVs of its colour
// (and z parity) change and none of them is in another's tile, so the phase-start answer equals
// the visit-start one.  The update kernel's task fetch then accounts flagged tasks exactly as a
// skipped visit (k_icd_sv fetch_task) without loading their tiles.  A warp per task (grid-stride).
__global__ void k_zero_flags(const int* __restrict__ flat, const int* __restrict__ brange,
                             const float* __restrict__ x, int nx, int ny, int nz_local, int z_offset,
                             int nz_total, int side, int nsvx, int nnb, int* __restrict__ keep)
{
    const int lane = threadIdx.x & 31;
    const int nwarps = gridDim.x * (blockDim.x >> 5), n = brange[1];
    for (int t = blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); t < n; t += nwarps) {
    const int tk = flat[t];
    const int z = tk >> 14, sv = tk & 16383;
    const int gx0 = (sv % nsvx) * side - 1, gy0 = (sv / nsvx) * side - 1;
    const int TW = side + 2, nzt = nnb == 26 ? 3 : 1;
    const size_t plane = (size_t)nx * ny;
    bool nz = false;
    for (int i = lane; i < nzt * TW * TW && !nz; i += 32) {
        const int tz = nzt == 3 ? i / (TW * TW) - 1 : 0, r = i % (TW * TW);
        const int gx = gx0 + r % TW, gy = gy0 + r / TW, gz = z_offset + z + tz;
        if (gx < 0 || gx >= nx || gy < 0 || gy >= ny || gz < 0 || gz >= nz_total) continue;
        nz = x[(size_t)(z + 1 + tz) * plane + (size_t)gy * nx + gx] != 0.f;
    }
    nz = __any_sync(0xffffffffu, nz);
    if (lane == 0) keep[t] = nz ? 1 : 0;
    }
}

__global__ void k_rmse(const float* __restrict__ x, const float* __restrict__ g, int64_t n,
                       double* acc)
{
    double s = 0.0;
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n;
         i += (int64_t)gridDim.x * blockDim.x) {
        const double d = (double)x[i] - (double)g[i];
        s += d * d;
    }
    for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
    if ((threadIdx.x & 31) == 0) atomicAdd(acc, s);
}

__global__ void k_finite(const float* __restrict__ a, int64_t n, int nonneg, int* flag)
{
    int bad = 0;
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n;
         i += (int64_t)gridDim.x * blockDim.x) {
        const float v = a[i];
        if (!isfinite(v) || (nonneg && v < 0.f)) bad = 1;
    }
    if (__any_sync(0xffffffffu, bad) && (threadIdx.x & 31) == 0) atomicOr(flag, 1);
}

}  // namespace

cudaError_t launch_select(const SchedParams& sp, cudaStream_t st)
{
    const int smem = sp.nsv_pad * 8;
    cudaError_t e = cudaFuncSetAttribute(k_select, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    if (e != cudaSuccess) return e;
    k_select<<<sp.nz_local, kSelThreads, smem, st>>>(sp);
    return cudaGetLastError();
}

cudaError_t launch_flatten(const int* task_list, const int* task_count, int nz_local, int z_offset,
                           int parities, int max_group, int batch, int thr, int nb, int* flat,
                           int* brange, cudaStream_t st)
{
    k_flatten<<<parities * 4, 256, 0, st>>>(task_list, task_count, nz_local, z_offset, parities,
                                            max_group, batch, thr, nb, flat, brange);
    return cudaGetLastError();
}

cudaError_t launch_zero_flags(const int* flat, const int* brange, const float* x, int nx, int ny,
                              int nz_local, int z_offset, int nz_total, int side, int nsvx, int nnb,
                              int max_tasks, int* keep, cudaStream_t st)
{
    if (max_tasks <= 0) return cudaSuccess;
    k_zero_flags<<<min((max_tasks + 7) / 8, 296), 256, 0, st>>>(flat, brange, x, nx, ny, nz_local, z_offset,
                                                                nz_total, side, nsvx, nnb, keep);
    return cudaGetLastError();
}

cudaError_t launch_rmse_partial(const float* x, const float* g, int64_t n, double* acc,
                                cudaStream_t st)
{
    k_rmse<<<296, 256, 0, st>>>(x, g, n, acc);
    return cudaGetLastError();
}

cudaError_t launch_check_finite(const float* a, int64_t n, int nonneg, int* flag, cudaStream_t st)
{
    k_finite<<<296, 256, 0, st>>>(a, n, nonneg, flag);
    return cudaGetLastError();
}

}  // namespace mbir
