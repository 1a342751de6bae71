// System-matrix precompute, compressed per SuperVoxel.
//
// Paper: A "encodes the CT equipment geometry"; it is stored sparse with a per-(voxel,
// view) start location, transformed into zero-padded chunks matched to the SV buffer
// (P:241-245), and quantised to one byte per entry with a per-voxel maximum.
//
// B200 design: for every (SV s, voxel slot v, view k) we keep the
// 8-bit offset of the voxel's first channel inside the SV's band at view k plus K = 4 uint8
// codes packed in one 32-bit word (or a float4 in fp32 mode).  Threads of the update kernel
// own views, so consecutive threads read consecutive 4-byte words: one 128-byte line per warp.
//
// Values are computed in double with -fmad=false (this TU), in the same arithmetic order for
// the channel index range as the oracle, so the integer index structure is bit-exact
// (reading R5).  The value itself uses the antiderivative of the pixel's trapezoidal shadow,
// an independent formulation from the oracle's polygon clipping (reading R4).
#include "mbir_internal.h"

namespace mbir {

namespace {

constexpr double kEps = 1e-9;  // channel-index guard, reading R5

// Antiderivative of the pixel shadow (chord length vs detector coordinate): trapezoid with
// plateau half-width h1, support half-width h2, peak P, total area d2 = dxy^2.
__device__ __forceinline__ double shadow_cdf(double tau, double h1, double h2, double P,
                                             double d2)
{
    if (tau <= -h2) return 0.0;
    if (tau >= h2) return d2;
    const double r = h2 - h1;
    if (tau < -h1) return P * (tau + h2) * (tau + h2) / (2.0 * r);
    if (tau <= h1) return 0.5 * P * r + P * (tau + h1);
    return d2 - P * (h2 - tau) * (h2 - tau) / (2.0 * r);
}

struct Col {
    int first, count;
    double v[kK];
};

// One (voxel, view) entry of A: channel range and strip areas / dchannel.
__device__ __forceinline__ Col column_entry(int nx, int ny, double d, int M, double dc,
                                            double center_offset, double c, double s, int ix,
                                            int iy)
{
    Col out;
    const double cx = ((double)ix - 0.5 * (double)(nx - 1)) * d;
    const double cy = ((double)iy - 0.5 * (double)(ny - 1)) * d;
    const double t0 = -0.5 * (double)M * dc + center_offset * dc;
    const double tj = cx * c + cy * s;
    const double ac = fabs(c), as = fabs(s);
    const double h2 = 0.5 * d * (ac + as);
    int f = (int)floor((tj - h2 - t0) / dc + kEps);
    int l = (int)ceil((tj + h2 - t0) / dc - kEps) - 1;
    if (f < 0) f = 0;
    if (l > M - 1) l = M - 1;
    int n = l - f + 1;
    if (n < 0) n = 0;
    out.first = (n > 0) ? f : 0;
    out.count = n;
    const double h1 = 0.5 * d * fabs(ac - as);
    const double P = d / fmax(ac, as);
    const double d2 = d * d;
#pragma unroll
    for (int i = 0; i < kK; ++i) {
        out.v[i] = 0.0;
        if (i < n) {
            const double lo = t0 + (double)(f + i) * dc, hi = lo + dc;
            out.v[i] = (shadow_cdf(hi - tj, h1, h2, P, d2) - shadow_cdf(lo - tj, h1, h2, P, d2)) / dc;
        }
    }
    return out;
}

constexpr int kColThreads = 256;
constexpr int kMaxViewsPerThread = 4;  // V <= 1024

// grid (S2, nsv): one block per (SV, slot) voxel; threads over views.
__global__ void __launch_bounds__(kColThreads) k_columns(
    int nx, int ny, double d, int V, int M, double dc, double center_offset,
    const double2* __restrict__ cs, int side, int nsvx, bool quantize, int32_t* __restrict__ first_tmp,
    DevA A, int* err)
{
    const int slot = blockIdx.x, sv = blockIdx.y;
    const int bx = sv % nsvx, by = sv / nsvx;
    const int ix = bx * side + slot % side, iy = by * side + slot / side;
    const bool valid = ix < nx && iy < ny;
    const size_t base = ((size_t)sv * A.S2 + slot) * A.VA;
    Col col[kMaxViewsPerThread];
    double amax = 0.0;
#pragma unroll
    for (int t = 0; t < kMaxViewsPerThread; ++t) {
        const int k = threadIdx.x + t * kColThreads;
        col[t].first = 0;
        col[t].count = 0;
        if (k < V && valid) {
            const double2 a = cs[k];
            col[t] = column_entry(nx, ny, d, M, dc, center_offset, a.x, a.y, ix, iy);
            if (col[t].count > kK) atomicOr(err, 1);
#pragma unroll
            for (int i = 0; i < kK; ++i)
                if (i < col[t].count && col[t].v[i] > amax) amax = col[t].v[i];
        }
    }
    // block max of amax (per-voxel maximum)
    __shared__ double red[kColThreads / 32];
    for (int o = 16; o > 0; o >>= 1) amax = fmax(amax, __shfl_xor_sync(0xffffffffu, amax, o));
    if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = amax;
    __syncthreads();
    if (threadIdx.x < 32) {
        double m = threadIdx.x < kColThreads / 32 ? red[threadIdx.x] : 0.0;
        for (int o = 16; o > 0; o >>= 1) m = fmax(m, __shfl_xor_sync(0xffffffffu, m, o));
        if (threadIdx.x == 0) red[0] = m;
    }
    __syncthreads();
    amax = red[0];
    if (threadIdx.x == 0) A.scale[(size_t)sv * A.S2 + slot] = quantize ? (float)(amax / 255.0) : 1.0f;
#pragma unroll
    for (int t = 0; t < kMaxViewsPerThread; ++t) {
        const int k = threadIdx.x + t * kColThreads;
        if (k >= V) continue;
        const int n = col[t].count < kK ? col[t].count : kK;
        first_tmp[base + apos(k, A.vpt)] = n > 0 ? col[t].first : -1;
        A.count[base + apos(k, A.vpt)] = (uint8_t)n;
        if (quantize) {
            uint32_t word = 0;
#pragma unroll
            for (int i = 0; i < kK; ++i) {
                // P:267-269, reading R6: (uint8) floor(A / amax * 255 + 0.5)
                uint32_t code = (i < n && amax > 0.0)
                                    ? (uint32_t)(uint8_t)floor(col[t].v[i] / amax * 255.0 + 0.5)
                                    : 0u;
                word |= code << (8 * i);
            }
            A.codes[base + apos(k, A.vpt)] = word;
        } else {
            A.vals[base + apos(k, A.vpt)] = make_float4((float)col[t].v[0], (float)col[t].v[1],
                                           (float)col[t].v[2], (float)col[t].v[3]);
        }
    }
}

// grid (nsv), threads over views: SV band [start, start + width) per view (Fig. 2).
__global__ void k_bands(int V, int S2, const int32_t* __restrict__ first_tmp, DevA A,
                        int* maxrow, int* maxwidth, int* err)
{
    const int sv = blockIdx.x;
    for (int k = threadIdx.x; k < V; k += blockDim.x) {
        int lo = 1 << 30, hi = -1;
        for (int v = 0; v < S2; ++v) {
            const size_t i = ((size_t)sv * S2 + v) * A.VA + apos(k, A.vpt);
            const int f = first_tmp[i];
            if (f < 0) continue;
            lo = min(lo, f);
            hi = max(hi, f + (int)A.count[i]);
        }
        if (hi < 0) lo = hi = 0;
        A.band_start[(size_t)sv * V + k] = lo;
        const int wdt = hi - lo;
        if (wdt > 255) atomicOr(err, 2);
        A.band_width[(size_t)sv * V + k] = (uint8_t)min(wdt, 255);
        atomicMax(maxwidth, wdt);
        int rowmax = 0;
        for (int v = 0; v < S2; ++v) {
            const size_t i = ((size_t)sv * S2 + v) * A.VA + apos(k, A.vpt);
            const int f = first_tmp[i];
            const int o = f < 0 ? 0 : f - lo;
            if (o > 255) atomicOr(err, 2);
            A.off[i] = (uint8_t)min(o, 255);
            rowmax = max(rowmax, o + kK);  // the kernel reads rows o .. o+K-1
        }
        atomicMax(maxrow, rowmax);
    }
}

// Plain-layout export of A (test hook): [ny*nx][V] first/count, [ny*nx][V][K] values/codes.
__global__ void k_export(int nx, int ny, double d, int V, int M, double dc, double center_offset,
                         const double2* __restrict__ cs, int side, int nsvx, DevA A,
                         const int64_t* __restrict__ vox, int32_t* first, int32_t* count,
                         float* vals, uint8_t* codes, float* scales, bool quantize)
{
    const int j = vox ? (int)vox[blockIdx.x] : (int)blockIdx.x;  // iy*nx + ix
    const size_t jo = blockIdx.x;                                   // output row
    const int ix = j % nx, iy = j / nx;
    const int sv = (iy / side) * nsvx + ix / side;
    const int slot = (iy % side) * side + ix % side;
    const size_t base = ((size_t)sv * A.S2 + slot) * A.VA;
    for (int k = threadIdx.x; k < V; k += blockDim.x) {
        const int n = A.count[base + apos(k, A.vpt)];
        const size_t o = jo * V + k;
        if (first) first[o] = n > 0 ? A.band_start[(size_t)sv * V + k] + A.off[base + apos(k, A.vpt)] : 0;
        if (count) count[o] = n;
        if (codes) {
            const uint32_t wd = quantize ? A.codes[base + apos(k, A.vpt)] : 0u;
            for (int i = 0; i < kK; ++i) codes[o * kK + i] = (uint8_t)(wd >> (8 * i));
        }
        if (vals) {
            // the values the update kernel uses: the stored fp32 entries, or (uint8 A) the
            // dequantised codes code * scale
            if (quantize) {
                const uint32_t wd = A.codes[base + apos(k, A.vpt)];
                const float sc = A.scale[(size_t)sv * A.S2 + slot];
                for (int i = 0; i < kK; ++i) vals[o * kK + i] = (float)((wd >> (8 * i)) & 255u) * sc;
            } else {
                const float4 v = A.vals[base + apos(k, A.vpt)];
                vals[o * kK + 0] = v.x;
                vals[o * kK + 1] = v.y;
                vals[o * kK + 2] = v.z;
                vals[o * kK + 3] = v.w;
            }
        }
    }
    if (scales && threadIdx.x == 0) scales[jo] = A.scale[(size_t)sv * A.S2 + slot];
}

}  // namespace

cudaError_t build_sysmatrix(const mbir_geometry& g, const double* d_angles_cs, int side, int nsvx,
                            int nsvy, bool quantize, DevA& A, int* d_err, int* d_maxrow,
                            cudaStream_t st)
{
    const size_t n = (size_t)A.nsv * A.S2 * A.VA;
    int32_t* first_tmp = nullptr;
    cudaError_t e = cudaMallocAsync(&first_tmp, n * sizeof(int32_t), st);
    if (e != cudaSuccess) return e;
    dim3 grid(A.S2, A.nsv);
    k_columns<<<grid, kColThreads, 0, st>>>(g.nx, g.ny, g.dxy, g.nviews, g.nchannels, g.dchannel,
                                            g.center_offset, (const double2*)d_angles_cs, side,
                                            nsvx, quantize, first_tmp, A, d_err);
    e = cudaGetLastError();
    if (e == cudaSuccess) {
        k_bands<<<A.nsv, 256, 0, st>>>(g.nviews, A.S2, first_tmp, A, d_maxrow, d_maxrow + 1, d_err);
        e = cudaGetLastError();
    }
    cudaFreeAsync(first_tmp, st);
    (void)nsvy;
    return e;
}

cudaError_t launch_export_sysmatrix(const DevA& A, int nx, int ny, int side, int nsvx,
                                    const int64_t* vox, int nvox, int32_t* first, int32_t* count,
                                    float* vals, uint8_t* codes, float* scales,
                                    const mbir_geometry& g, const double* d_angles_cs,
                                    cudaStream_t st)
{
    const int n = vox ? nvox : nx * ny;
    k_export<<<n, 256, 0, st>>>(nx, ny, g.dxy, g.nviews, g.nchannels, g.dchannel,
                                g.center_offset, (const double2*)d_angles_cs, side, nsvx, A, vox,
                                first, count, vals, codes, scales, A.codes != nullptr);
    return cudaGetLastError();
}

}  // namespace mbir
