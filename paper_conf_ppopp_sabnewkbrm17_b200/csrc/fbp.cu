// Filtered back-projection initial image (mbir_init_fbp).  Not part of the paper's method: the
// paper never states its initial image (reading R23); ICD converges from any x0, and a
// start near the MAP point shortens the first sweeps, whose SV blocks otherwise absorb whole ray
// sums from x0 = 0.  Textbook parallel-beam FBP (Kak & Slaney, "Principles of Computerized
// Tomographic Imaging", ch. 3, eqs. 61-63): Ram-Lak filter by direct convolution in the channel
// domain, then linearly interpolated back-projection over the views, clipped at 0 with
// positivity (reading R3).  Setup-time kernels (one launch each per call).
#include "mbir_internal.h"

namespace mbir {

namespace {

constexpr int kRampThreads = 256;

// q[z][k][m] = dc * sum_n h(m - n) p[z][k][n],  h(0) = 1/(4 dc^2), h(d) = -1/(pi^2 d^2 dc^2) for
// odd d, 0 for even d != 0 (band-limited ramp sampled at the channel pitch).  One block per
// (view, slice) row, the row staged in shared memory.
__global__ void __launch_bounds__(kRampThreads) k_ramp(const float* __restrict__ p, float* __restrict__ q,
                                                       int M, double dc)
{
    extern __shared__ float row[];  // [M] the projection row, then [M/2 + 1] weights 1/d^2, d odd
    float* wt = row + M;
    const size_t base = ((size_t)blockIdx.y * gridDim.x + blockIdx.x) * M;
    for (int i = threadIdx.x; i < M; i += blockDim.x) row[i] = p[base + i];
    for (int i = threadIdx.x; i <= M / 2; i += blockDim.x) {
        const float d = (float)(2 * i + 1);
        wt[i] = 1.f / (d * d);
    }
    __syncthreads();
    const float inv_pi2 = (float)(1.0 / (3.14159265358979323846 * 3.14159265358979323846));
    for (int m = threadIdx.x; m < M; m += blockDim.x) {
        float acc = 0.25f * row[m];
        float odd = 0.f;
        for (int d = 1; d < M; d += 2) {
            const float a = (m - d >= 0 ? row[m - d] : 0.f) + (m + d < M ? row[m + d] : 0.f);
            odd = fmaf(a, wt[d >> 1], odd);
        }
        acc -= inv_pi2 * odd;
        q[base + m] = acc * (float)(1.0 / dc);  // dc * h, h ~ 1/dc^2
    }
}

// x[z][iy][ix] = (pi / V) sum_k q[z][k](t),  t = x cos(theta_k) + y sin(theta_k), channel m covering
// [t0 + m dc, t0 + (m+1) dc), linear interpolation between channel centres, 0 outside.
__global__ void k_backproject(const float* __restrict__ q, const double2* __restrict__ cs, float* __restrict__ x,
                              int nx, int ny, int V, int M, double dxy, double dc, double t0,
                              float scale, int positivity)
{
    const int ix = blockIdx.x * blockDim.x + threadIdx.x;
    const int iy = blockIdx.y * blockDim.y + threadIdx.y;
    const int z = blockIdx.z;
    if (ix >= nx || iy >= ny) return;
    const double xc = (ix - 0.5 * (nx - 1)) * dxy, yc = (iy - 0.5 * (ny - 1)) * dxy;
    const double inv_dc = 1.0 / dc;
    const float* qz = q + (size_t)z * V * M;
    float acc = 0.f;
    for (int k = 0; k < V; ++k) {
        const double2 c = cs[k];
        // channel-centre coordinate (double FMAs, no per-sample division)
        const float u = (float)(fma(xc, c.x, fma(yc, c.y, -t0)) * inv_dc) - 0.5f;
        const float fl = floorf(u);
        const int m = (int)fl;
        const float f = u - fl;
        const float* row = qz + (size_t)k * M;
        const float a = (m >= 0 && m < M) ? __ldg(row + m) : 0.f;
        const float b = (m + 1 >= 0 && m + 1 < M) ? __ldg(row + m + 1) : 0.f;
        acc += fmaf(f, b - a, a);
    }
    float v = acc * scale;
    if (positivity) v = fmaxf(v, 0.f);
    x[((size_t)z * ny + iy) * nx + ix] = v;
}

}  // namespace

cudaError_t launch_fbp(const mbir_geometry& g, const double* d_cs, const float* y, float* q, float* x,
                       int positivity, cudaStream_t st)
{
    const int V = g.nviews, M = g.nchannels;
    const size_t smem = (size_t)(M + M / 2 + 1) * sizeof(float);
    if (smem > 48 * 1024) {
        cudaError_t e = cudaFuncSetAttribute(k_ramp, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        if (e != cudaSuccess) return e;
    }
    k_ramp<<<dim3(V, g.nz_local), kRampThreads, smem, st>>>(y, q, M, g.dchannel);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return e;
    const double t0 = -0.5 * M * g.dchannel + g.center_offset * g.dchannel;
    const dim3 blk(32, 8), grd((g.nx + 31) / 32, (g.ny + 7) / 8, g.nz_local);
    k_backproject<<<grd, blk, 0, st>>>(q, (const double2*)d_cs, x, g.nx, g.ny, V, M, g.dxy, g.dchannel, t0,
                                       (float)(3.14159265358979323846 / V), positivity);
    return cudaGetLastError();
}

}  // namespace mbir
