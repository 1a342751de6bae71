// Setup-time and test-hook kernels that share the update kernel's data layout (svicd.cu):
// theta2 = A^T W A per (slice, voxel) (Alg1:6, fixed by w), e = y - A x for warm starts, and
// the fixed-state probe of Alg. 1 steps 1-7 (test hook).
#include "mbir_internal.h"

namespace mbir {

namespace {

constexpr unsigned kFull = 0xffffffffu;

// phi(D) = rho'(D)/(2D) for the q-GGMRF potential with q = 2 (reading R1)
__device__ __forceinline__ float phi_f(const PriorConst& pc, float d)
{
    const float ad = fabsf(d);
    float u;
    if (pc.qmp == 0.f)
        u = 1.f;
    else
        u = (ad == 0.f) ? 0.f : exp2f(pc.qmp * __log2f(ad * pc.inv_Ts));
    const float opu = 1.f + u;
    return __fdividef(pc.c_phi * (pc.pq + u), opu * opu);
}

// uint8 code i of a packed word -> float, via the 2^23 magic (PRMT + FADD, no I2F)
__device__ __forceinline__ float dq(uint32_t word, int i)
{
    const uint32_t b = __byte_perm(word, 0x4B000000u, 0x7440u | (uint32_t)i);
    return __uint_as_float(b) - 8388608.f;
}

__device__ __forceinline__ void red_add_f32(float* p, float v)
{
    asm volatile("red.global.add.f32 [%0], %1;" ::"l"(p), "f"(v));
}

// theta2[z][sv][slot] = sum_k sum_i w * A^2 (Alg1:6), fixed for a given sinogram.  One block per
// (SV, slice), one warp per voxel; lanes walk the voxel's A record positions (coalesced) and
// read w through the read-only path (the SV's band is L1/L2-resident).  Setup-time kernel.
template <bool U8>
__global__ void k_theta2(const IcdParams P)
{
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nw = blockDim.x >> 5;
    const int z = blockIdx.x, sv = blockIdx.y;
    const float* wz = P.w + (size_t)z * P.V * P.M;
    const int vpt = P.A.vpt;
    for (int slot = warp; slot < P.S2; slot += nw) {
        const size_t ab = ((size_t)sv * P.S2 + slot) * P.A.VA;
        const float sc = P.A.scale[(size_t)sv * P.S2 + slot];
        float acc = 0.f;
#pragma unroll 4
        for (int pk = lane; pk < P.A.VA; pk += 32) {  // record positions, coalesced (4 in flight)
            const int qq = pk / vpt, t = pk % vpt;     // inverse of apos()
            const int k = min(((qq >> 5) * vpt + t) * 32 + (qq & 31), P.V - 1);  // padded: count 0
            const int n = P.A.count[ab + pk];
            const int o = P.A.band_start[(size_t)sv * P.V + k] + P.A.off[ab + pk];
            float a[4];
            if (U8) {
                const uint32_t c = P.A.codes[ab + pk];
                for (int i = 0; i < 4; ++i) a[i] = dq(c, i) * sc;
            } else {
                const float4 q = P.A.vals[ab + pk];
                a[0] = q.x; a[1] = q.y; a[2] = q.z; a[3] = q.w;
            }
            for (int i = 0; i < 4; ++i)
                if (i < n) acc += __ldg(wz + (size_t)k * P.M + o + i) * a[i] * a[i];
        }
        for (int o = 16; o > 0; o >>= 1) acc += __shfl_xor_sync(kFull, acc, o);
        if (lane == 0) P.theta2[((size_t)z * P.nsv + sv) * P.S2 + slot] = acc;
    }
}

// e[z] += -A x[z] for one (slice, SV) per block (e must hold y on entry).  Threads own views;
// accumulates the SV's band in smem, then adds it to e atomically.  Setup-time kernel.
template <bool U8>
__global__ void k_forward(const IcdParams P)
{
    extern __shared__ __align__(16) unsigned char smem[];
    float* acc = (float*)smem;  // [rows][Vs]
    const int z = blockIdx.x, sv = blockIdx.y;
    const int bx = sv % P.nsvx, by = sv / P.nsvx;
    const int gx0 = bx * P.side, gy0 = by * P.side;
    const int tw = min(P.side, P.nx - gx0), th = min(P.side, P.ny - gy0);
    const size_t plane = (size_t)P.nx * P.ny;
    float* xs = acc + P.rows * P.Vs;  // [S2] the SV's voxel values
    bool nz = false;
    for (int slot = threadIdx.x; slot < P.S2; slot += blockDim.x) {
        const int lx = slot % P.side, ly = slot / P.side;
        const float xv = (lx < tw && ly < th) ? P.x[(size_t)(z + 1) * plane + (size_t)(gy0 + ly) * P.nx + gx0 + lx] : 0.f;
        xs[slot] = xv;
        nz |= xv != 0.f;
    }
    if (!__syncthreads_or(nz)) return;  // all-zero SV contributes nothing
    for (int i = threadIdx.x; i < P.rows * P.Vs; i += blockDim.x) acc[i] = 0.f;
    __syncthreads();
    bool any = false;
    for (int k = threadIdx.x; k < P.V; k += blockDim.x) {
        for (int slot = 0; slot < P.S2; ++slot) {
            const float xv = xs[slot];
            if (xv == 0.f) continue;
            any = true;
            const size_t ai = ((size_t)sv * P.S2 + slot) * P.A.VA + apos(k, P.A.vpt);
            const int o = P.A.off[ai];
            const float sc = P.A.scale[(size_t)sv * P.S2 + slot];
            for (int i = 0; i < 4; ++i) {
                float a;
                if (U8) {
                    a = dq(P.A.codes[ai], i) * sc;
                } else {
                    const float4 q = P.A.vals[ai];
                    a = i == 0 ? q.x : i == 1 ? q.y : i == 2 ? q.z : q.w;
                }
                acc[(o + i) * P.Vs + k] += a * xv;
            }
        }
    }
    if (!__syncthreads_or(any)) return;
    float* ez = P.e + (size_t)z * P.V * P.M;
    for (int k = threadIdx.x; k < P.V; k += blockDim.x) {
        const int bs = P.A.band_start[(size_t)sv * P.V + k];
        const int bw = P.A.band_width[(size_t)sv * P.V + k];
        for (int c = 0; c < bw; ++c) {
            const float d = acc[c * P.Vs + k];
            if (d != 0.f) red_add_f32(ez + (size_t)k * P.M + bs + c, -d);
        }
    }
}

// Alg. 1 steps 1-7 for given voxels at the current state, from GLOBAL e/w/x (test hook).
template <bool U8>
__global__ void k_probe(const IcdParams P, const int64_t* vox, float* out3)
{
    const int q = blockIdx.x;
    const int64_t j = vox[q];
    const size_t plane = (size_t)P.nx * P.ny;
    const int z = (int)(j / plane);
    const int iy = (int)((j % plane) / P.nx), ix = (int)(j % P.nx);
    const int sv = (iy / P.side) * P.nsvx + ix / P.side;
    const int slot = (iy % P.side) * P.side + ix % P.side;
    const size_t ab = ((size_t)sv * P.S2 + slot) * P.A.VA;
    const float sc = P.A.scale[(size_t)sv * P.S2 + slot];
    const float* wz = P.w + (size_t)z * P.V * P.M;
    const float* ez = P.e + (size_t)z * P.V * P.M;
    float t1 = 0.f, t2 = 0.f;
    for (int k = threadIdx.x; k < P.V; k += blockDim.x) {
        const int f = P.A.band_start[(size_t)sv * P.V + k] + P.A.off[ab + apos(k, P.A.vpt)];
        const int n = P.A.count[ab + apos(k, P.A.vpt)];
        for (int i = 0; i < 4 && i < n; ++i) {
            float a;
            if (U8) {
                a = dq(P.A.codes[ab + apos(k, P.A.vpt)], i) * sc;
            } else {
                const float4 v4 = P.A.vals[ab + apos(k, P.A.vpt)];
                a = i == 0 ? v4.x : i == 1 ? v4.y : i == 2 ? v4.z : v4.w;
            }
            const float ww = wz[(size_t)k * P.M + f + i];
            t1 -= ww * a * ez[(size_t)k * P.M + f + i];
            t2 += ww * a * a;
        }
    }
    __shared__ float r1[32], r2[32];
    for (int o = 16; o > 0; o >>= 1) {
        t1 += __shfl_xor_sync(kFull, t1, o);
        t2 += __shfl_xor_sync(kFull, t2, o);
    }
    if ((threadIdx.x & 31) == 0) {
        r1[threadIdx.x >> 5] = t1;
        r2[threadIdx.x >> 5] = t2;
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        float T1 = 0.f, T2 = 0.f;
        for (int w = 0; w < (int)(blockDim.x >> 5); ++w) {
            T1 += r1[w];
            T2 += r2[w];
        }
        const float v = P.x[(size_t)(z + 1) * plane + (size_t)iy * P.nx + ix];
        float sbv = 0.f, sbx = 0.f;
        const int zg = P.z_offset + z;
        for (int r = 0; r < P.pc.nnb; ++r) {
            const int gx = ix + P.pc.dx[r], gy = iy + P.pc.dy[r], gz = zg + P.pc.dz[r];
            if (gx < 0 || gx >= P.nx || gy < 0 || gy >= P.ny || gz < 0 || gz >= P.nz_total) continue;
            const float xr = P.x[(size_t)(z + 1 + P.pc.dz[r]) * plane + (size_t)gy * P.nx + gx];
            const float bt = P.pc.b[r] * phi_f(P.pc, v - xr);
            sbv += bt;
            sbx += bt * xr;
        }
        const float num = T2 * v - T1 + 2.f * sbx, den = T2 + 2.f * sbv;
        float u = den > 0.f ? num / den : v;
        if (P.pc.positivity) u = fmaxf(u, 0.f);
        out3[3 * q] = T1;
        out3[3 * q + 1] = T2;
        out3[3 * q + 2] = u - v;
    }
}

}  // namespace

cudaError_t launch_theta2(const IcdParams& p, bool quantize, cudaStream_t st)
{
    auto k = quantize ? k_theta2<true> : k_theta2<false>;
    k<<<dim3(p.nz_local, p.nsv), 512, 0, st>>>(p);  // slices of one SV adjacent: A from L2
    return cudaGetLastError();
}

cudaError_t launch_forward(const IcdParams& p, bool quantize, const float* y, cudaStream_t st)
{
    cudaError_t e = cudaMemcpyAsync(p.e, y, sizeof(float) * (size_t)p.nz_local * p.V * p.M,
                                    cudaMemcpyDeviceToDevice, st);
    if (e != cudaSuccess) return e;
    const int smem = (p.rows * p.Vs + p.S2) * 4;
    auto k = quantize ? k_forward<true> : k_forward<false>;
    e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    if (e != cudaSuccess) return e;
    k<<<dim3(p.nz_local, p.nsv), 256, smem, st>>>(p);  // slices of one SV adjacent: A from L2
    return cudaGetLastError();
}

cudaError_t launch_probe(const IcdParams& p, bool quantize, int nnb, const int64_t* vox, int n,
                         float* out3, cudaStream_t st)
{
    (void)nnb;
    if (quantize)
        k_probe<true><<<n, 256, 0, st>>>(p, vox, out3);
    else
        k_probe<false><<<n, 256, 0, st>>>(p, vox, out3);
    return cudaGetLastError();
}

}  // namespace mbir
