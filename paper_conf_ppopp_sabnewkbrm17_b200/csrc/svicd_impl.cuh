// The fused SuperVoxel ICD update kernel for sm_100a.  Included by
// svicd.cu (host-side layout and dispatch) and by the four instantiating translation units
// svicd_n{8,26}_{u8,f32}.cu.
//
// Paper: Alg. 1 is the per-voxel update; Alg. 3 runs it with
// intra-voxel, intra-SV and inter-SV parallelism over SV buffers
// created before and written back after the update.
//
// B200 design.  One CTA per SM owns one (slice, SV) task at a time and
// pulls tasks from the phase list (persistent grid).  Its warps have three roles:
//   * nvw VIEW warps: view warp w, lane l owns views (w*VPT + t)*32 + l, t < VPT.  The SV buffer
//     (e and w over the SV's sinogram band) lives in shared memory as rows
//     [channel offset in band] x [view], e and w rows interleaved (row r of e, then row r of w),
//     with a row length that is a multiple of 32 views, so a warp's 32 lanes hit 32 distinct
//     banks for any per-view offsets: conflict-free gathers and scatters, no atomics (a thread is
//     the only writer of its views).
//   * the DELTA warp derives each voxel's delta (Alg1:7-8, q-GGMRF surrogate, reading R1) from
//     the view warps' partial sums and the surrogate terms, and writes the new value into the
//     shared-memory x tile;
//   * the PRIOR warp computes the next voxel's surrogate terms from the x tile (one neighbour per
//     lane) while the current voxel is in flight, with the previous voxel's OLD value; the delta
//     warp replaces that one neighbour's term once the new value is known (exact).
// Voxels of the SV are updated in a random order exactly as sequential ICD, one per step: the
// view warps gather theta1's partials of voxel i from e (holding voxel i - 1's scatter), prepare
// voxel i + 1 (A record from the cp.async ring, dequantised; w*A in registers) while the delta
// is derived, then scatter voxel i into their own views.  A records (uint8 codes + band offsets)
// are streamed R voxels ahead by per-thread cp.async.  theta2 = A^T W A is stored per (slice,
// voxel); the first iteration after new weights reduces it here (T2) alongside theta1.  The
// write-back is delta e = final - e_init per aligned band window with red.global.add.v4.f32
// (same-colour SVs share sinogram entries).  The next task's inputs are prepared
// while the current one runs.
#pragma once
#include "mbir_internal.h"

#include <map>
#include <mutex>

namespace mbir {

namespace {

constexpr unsigned kFull = 0xffffffffu;

// phi(D) = rho'(D)/(2D) for the q-GGMRF potential with q = 2 (reading R1):
//   phi = c_phi * (q/p + u) / (1 + u)^2,  u = |D/(T sigma)|^(q-p)   (|D|^(q-2) = 1)
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

// dequantised codes i, i + 1 of a packed word as a channel pair, via the 2^23 magic (2 PRMT +
// 1 FADD2, no I2F)
__device__ __forceinline__ float2 dq2(uint32_t word, int i)
{
    const float2 m = make_float2(__uint_as_float(__byte_perm(word, 0x4B000000u, 0x7440u | (uint32_t)i)),
                                 __uint_as_float(__byte_perm(word, 0x4B000000u, 0x7441u + (uint32_t)i)));
    return __fadd2_rn(m, make_float2(-8388608.f, -8388608.f));
}

// vector atomic add of 4 consecutive floats (16-byte aligned), sm_90+
__device__ __forceinline__ void red_add_v4(float* p, float a, float b, float c, float d)
{
    asm volatile("red.global.add.v4.f32 [%0], {%1, %2, %3, %4};" ::"l"(p), "f"(a), "f"(b), "f"(c), "f"(d)
                 : "memory");
}

__device__ __forceinline__ uint64_t mix64(uint64_t z)
{
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
    return z ^ (z >> 31);
}

__device__ __forceinline__ uint32_t smem_u32(const void* p)
{
    return (uint32_t)__cvta_generic_to_shared(p);
}
// per-thread asynchronous global -> shared copies (LDGSTS), tracked per thread by commit groups
__device__ __forceinline__ void cp_async16(void* dst, const void* src)
{
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(smem_u32(dst)), "l"(src) : "memory");
}
__device__ __forceinline__ void cp_async8(void* dst, const void* src)
{
    asm volatile("cp.async.ca.shared.global [%0], [%1], 8;" ::"r"(smem_u32(dst)), "l"(src) : "memory");
}
__device__ __forceinline__ void cp_async4(void* dst, const void* src)
{
    asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" ::"r"(smem_u32(dst)), "l"(src) : "memory");
}
// 4-byte copy that writes zeros instead when !valid (src_size 0)
__device__ __forceinline__ void cp_async4_zfill(void* dst, const void* src, bool valid)
{
    asm volatile("cp.async.ca.shared.global [%0], [%1], 4, %2;" ::"r"(smem_u32(dst)), "l"(src), "r"(valid ? 4 : 0) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_async_wait()
{
    asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory");
}
// ---- thread-block cluster (CL = 2: the two CTAs of a cluster split a task's views) ----
__device__ __forceinline__ uint32_t cluster_rank()
{
    uint32_t r;
    asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
    return r;
}
// shared::cluster address of the same shared-memory location in CTA `rank` of the cluster
__device__ __forceinline__ uint32_t peer_addr(const void* p, uint32_t rank)
{
    uint32_t a;
    asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(a) : "r"(smem_u32(p)), "r"(rank));
    return a;
}
__device__ __forceinline__ void st_peer_f32(uint32_t a, float v)
{
    asm volatile("st.shared::cluster.f32 [%0], %1;" ::"r"(a), "f"(v) : "memory");
}
__device__ __forceinline__ void st_peer_u32(uint32_t a, uint32_t v)
{
    asm volatile("st.shared::cluster.u32 [%0], %1;" ::"r"(a), "r"(v) : "memory");
}
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count)
{
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
// arrive on the peer CTA's mbarrier; release at cluster scope orders this thread's earlier
// st.shared::cluster writes before the arrival
__device__ __forceinline__ void mbar_arrive_peer(uint32_t a)
{
    asm volatile("mbarrier.arrive.release.cluster.shared::cluster.b64 _, [%0];" ::"r"(a) : "memory");
}
// wait for phase `parity` of a local mbarrier with acquire at cluster scope (sees the peer's
// released writes)
__device__ __forceinline__ void mbar_wait_cluster(uint64_t* bar, uint32_t parity)
{
    asm volatile(
        "{\n\t.reg .pred p;\n"
        "WAITC_%=:\n\t"
        "mbarrier.try_wait.parity.acquire.cluster.shared::cta.b64 p, [%0], %1;\n\t"
        "@!p bra WAITC_%=;\n}" ::"r"(smem_u32(bar)),
        "r"(parity)
        : "memory");
}
__device__ __forceinline__ void cluster_sync_all()
{
    asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}

// one 128-bit shared-memory load (kept vector: the staging row reads are conflict-free only as
// LDS.128; split into scalar loads they would be 4-way bank conflicts)
__device__ __forceinline__ float4 lds128(const float* p)
{
    float4 v;
    asm volatile("ld.shared.v4.f32 {%0, %1, %2, %3}, [%4];" : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "r"(smem_u32(p)));
    return v;
}
// named barriers: sync (wait for `n` threads incl. this one) / arrive (count and go on).  The
// non-.aligned forms: the role warps reach them right after lane-0-only work, and the aligned
// bar.sync / bar.arrive would require the warp to be converged there (compute-sanitizer synccheck)
__device__ __forceinline__ void bar_sync(int id, int n) { asm volatile("barrier.sync %0, %1;" ::"r"(id), "r"(n) : "memory"); }
__device__ __forceinline__ void bar_arrive(int id, int n) { asm volatile("barrier.arrive %0, %1;" ::"r"(id), "r"(n) : "memory"); }

// The prior warp's lane r owns neighbour r of the neighbourhood (reading R2): offset (dx, dy, dz),
// tile-index offset dt and weight w (0: no neighbour / lane r >= 26)
struct NbrOne {
    int dx, dy, dz, dt;
    float w;
};

// surrogate terms of voxel i of the visiting order, computed from the x tile in which the voxels
// of the previous step (voxel ip0 = i - 1, or with voxel pairs the previous pair ip0, ip1) still
// have their OLD values and every earlier update is applied: the sums s = sum_r b_r phi(v - x_r),
// sx = sum_r b_r phi(v - x_r) x_r (Alg1:7, reading R1; free boundary), v = x_i, and for each such
// previous voxel that is a neighbour of i its term (btu) and weight (bwu), which the delta warp
// replaces by the term at the new value: exact.  (With pairs, the other voxel of i's own pair
// keeps its old value: both are computed from the same state.)
struct __align__(16) PriTerm {
    float s, sx, v, btu0, bwu0, btu1, bwu1, pad;  // 32 B: read as two 16-byte words
};

template <int NP>  // previous-step voxels to report (1, or 2 with voxel pairs)
__device__ __forceinline__ void prior_one(const int* tof, int i, int ip0, int ip1, const float* xt, int cslot,
                                          int TW, int gx0, int gy0, int zg, const IcdParams& P, const NbrOne& nb,
                                          int lane, PriTerm* out)
{
    const int tv = tof[i];
    const int lx = tv & 255, ly = tv >> 8;
    const int c0 = cslot + ly * TW + lx;
    const float v = xt[c0];
    const int gx = gx0 + lx + nb.dx, gy = gy0 + ly + nb.dy, gz = zg + nb.dz;
    const bool ok = nb.w != 0.f && gx >= 0 && gx < P.nx && gy >= 0 && gy < P.ny && gz >= 0 && gz < P.nz_total;
    const float xr = xt[c0 + nb.dt];  // always inside the tile (its ring covers the neighbourhood)
    const float bt = ok ? nb.w * phi_f(P.pc, v - xr) : 0.f;
    float s = bt, sx = bt * xr;
    bool m0 = false, m1 = false;
    if (ip0 >= 0) {
        const int tu = tof[ip0];
        m0 = ok && nb.dz == 0 && nb.dx == (tu & 255) - lx && nb.dy == (tu >> 8) - ly;
    }
    if (NP == 2 && ip1 >= 0) {
        const int tu = tof[ip1];
        m1 = ok && nb.dz == 0 && nb.dx == (tu & 255) - lx && nb.dy == (tu >> 8) - ly;
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        s += __shfl_xor_sync(kFull, s, o);
        sx += __shfl_xor_sync(kFull, sx, o);
    }
    const unsigned w0 = __ballot_sync(kFull, m0);
    const int src0 = w0 ? __ffs(w0) - 1 : 0;
    const float btu0 = __shfl_sync(kFull, bt, src0), bwu0 = __shfl_sync(kFull, nb.w, src0);
    float btu1 = 0.f, bwu1 = 0.f;
    if (NP == 2) {
        const unsigned w1 = __ballot_sync(kFull, m1);
        const int src1 = w1 ? __ffs(w1) - 1 : 0;
        btu1 = __shfl_sync(kFull, bt, src1);
        bwu1 = __shfl_sync(kFull, nb.w, src1);
        if (!w1) btu1 = bwu1 = 0.f;
    }
    if (lane == 0) *out = PriTerm{s, sx, v, w0 ? btu0 : 0.f, w0 ? bwu0 : 0.f, btu1, bwu1, 0.f};
}

// sum of the view warps' partials (slots) in a fixed tree order (<= 8 or 16 slots)
template <bool N8>
__device__ __forceinline__ float slot_sum(const float* rq)
{
    const float4 r0 = *(const float4*)rq, r1 = *(const float4*)(rq + 4);
    float2 q = __fadd2_rn(__fadd2_rn(make_float2(r0.x, r0.y), make_float2(r0.z, r0.w)),
                          __fadd2_rn(make_float2(r1.x, r1.y), make_float2(r1.z, r1.w)));
    if (!N8) {
        const float4 r2 = *(const float4*)(rq + 8), r3 = *(const float4*)(rq + 12);
        q = __fadd2_rn(q, __fadd2_rn(__fadd2_rn(make_float2(r2.x, r2.y), make_float2(r2.z, r2.w)),
                                     __fadd2_rn(make_float2(r3.x, r3.y), make_float2(r3.z, r3.w))));
    }
    return q.x + q.y;
}

__host__ __device__ inline int align16(int b) { return (b + 15) & ~15; }

// row stride (floats) of a view warp's 32-row transpose staging tile: 16-byte rows, so a lane moves
// 4 window positions with one STS.128 / LDS.128; every quarter-warp (one shared-memory wavefront
// of a 128-bit access) then touches 8 distinct 4-bank groups, on the put and on the read
constexpr int kStg = 36;

// SV-buffer geometry: VS = view columns (compile-time: 4 views per lane x 6 warps, or 1 x 4),
// rows of e and w interleaved, so e row r sits at float offset 2 r VS and w row r at (2 r + 1) VS:
// a thread reaches all four channels of a voxel's record in both arrays with immediate offsets
// from one address
__host__ __device__ constexpr int svb_cols(int vpt, int cl = 1) { return (vpt == 1 ? 128 : 768) / cl; }

constexpr int kNSL = 16;  // partial-sum slots per quantity and step (>= view warps)

// the pack and the write-back move 32-view tiles; tile warp w (< VA / 128: the record stride VA
// is a multiple of 128) handles tiles 4w ... 4w + 3 whatever the voxel loop's view ownership
// (those phases are bracketed by CTA barriers), so the staging area is sized for <= 6 tile warps
constexpr int kTileW = 4;
__host__ __device__ constexpr int tile_warps(int va) { return va / (32 * kTileW); }

// threads per CTA: VPT 4 -> <= 6 view warps, VPT 3 -> <= 8, VPT 2 -> <= 12, VPT 1 -> <= 4;
// + the delta and prior warps
__host__ __device__ constexpr int max_threads(int vpt) { return vpt == 2 ? 448 : vpt == 3 ? 320 : 256; }

// named barriers of the voxel-loop protocol (0 is __syncthreads)
constexpr int kBarA = 1;  // the view warps' theta1 partials of a voxel are ready
constexpr int kBarB = 2;  // the delta warp has published the voxel's delta
constexpr int kBarX = 3;  // the delta warp has written the previous voxel's new value into the x tile
constexpr int kBarP = 4;  // task preparation steps (delta + prior warps)
constexpr int kBarT = 5;  // the prior warp's surrogate terms of a voxel are ready

// A-record stage: U8: codes u32[VA] then offsets u8[VA]; fp32: float4[VA] then offsets u8[VA]
__host__ __device__ inline SmemLayout svicd_layout(int rows, int side, int S2, int nnb, int VA, bool u8,
                                                   int nstage, int nvw, int vpt, int V, int cl = 1)
{
    VA /= cl;  // this CTA's record positions (and views)
    SmemLayout L;
    const int TW = side + 2;
    const int nzt = nnb == 26 ? 3 : 1;
    int o = 0;
    L.sb_e = o;  o = align16(o + 2 * rows * svb_cols(vpt, cl) * 4);  // e / w rows interleaved
    L.sb_w = L.sb_e + svb_cols(vpt, cl) * 4;
    L.xt = o;    o = align16(o + 2 * nzt * TW * TW * 4);  // [2 tasks]: current / next
    L.list = o;  o = align16(o + 2 * S2 * 4);
    L.flags = o; o = align16(o + S2 * 4);
    L.tof = o;   o = align16(o + 2 * S2 * 4);
    L.red = o;   o = align16(o + 2 * 2 * 2 * kNSL * 4);  // [2 steps][2 voxels][theta1, theta2][kNSL view warps]
    L.pri = o;   o = align16(o + 2 * 2 * (int)sizeof(PriTerm));  // [2 steps][2 voxels]
    L.vscale = o; o = align16(o + 2 * S2 * 4);
    L.vth2 = o;  o = align16(o + 2 * S2 * 4);
    L.misc = o;  o = align16(o + 16 * 4);
    L.off_in_stage = VA * (u8 ? 4 : 16);
    L.stage_bytes = align16(L.off_in_stage + VA);
    // the A-record ring (voxel loop) and the transpose staging tiles (pack, write-back) are never
    // live at the same time: they share one region
    L.astage = o;
    L.staging = o;
    o = align16(o + max(nstage * L.stage_bytes, tile_warps(VA) * 32 * kStg * 4));
    L.mbar = o;  o = align16(o + 5 * 32 * 4);  // neighbour tables [dx | dy | dz | b | tile offset][32]
    L.rscale = o; o = align16(o + S2 * 4);      // the next task's inputs as copied (cp.async):
    L.rth2 = o;  o = align16(o + S2 * 4);       //   per-slot scales and theta2,
    L.rbs = o;   o = align16(o + V * 4);        //   band start and width per view
    L.rbw = o;   o = align16(o + V);
    L.binfo = o; o = align16(o + 2 * VA * cl * 4);  // band (row offset << 6 | width) per view, 2 tasks
    L.cx = o;    o = align16(o + 2 * 2 * 2 * 4 + 4 * 8);  // CL = 2: partial sums [2 steps][2 quantities][2 CTAs], mbarriers
    L.total = o;
    return L;
}

// this thread's VPT adjacent records from a stage as raw words (CW = 1: a uint8 code word per
// view; CW = 4: fp32 values), and the band offsets packed in one word (VPT bytes)
template <int VPT, int CW>
__device__ __forceinline__ void load_words(const unsigned char* stg, int off_in_stage, int tp,
                                           uint32_t (&c)[VPT][CW], uint32_t& ob)
{
    if (CW == 1 && VPT == 4) {
        const uint4 c4 = ((const uint4*)stg)[tp];
        c[0][0] = c4.x;
        c[VPT > 1 ? 1 : 0][0] = c4.y;
        c[VPT > 2 ? 2 : 0][0] = c4.z;
        c[VPT > 3 ? 3 : 0][0] = c4.w;
    } else if (CW == 1 && VPT == 2) {
        const uint2 c2 = ((const uint2*)stg)[tp];
        c[0][0] = c2.x;
        c[VPT > 1 ? 1 : 0][0] = c2.y;
    } else {
#pragma unroll
        for (int t = 0; t < VPT; ++t) {
            if (CW == 4) {
                const uint4 v = ((const uint4*)stg)[tp * VPT + t];
                c[t][0] = v.x;
                c[t][CW > 1 ? 1 : 0] = v.y;
                c[t][CW > 2 ? 2 : 0] = v.z;
                c[t][CW > 3 ? 3 : 0] = v.w;
            } else {
                c[t][0] = ((const uint32_t*)stg)[tp * VPT + t];
            }
        }
    }
    if (VPT == 4) ob = ((const uint32_t*)(stg + off_in_stage))[tp];
    if (VPT == 3) {
        const unsigned char* o3 = stg + off_in_stage + 3 * tp;
        ob = (uint32_t)o3[0] | ((uint32_t)o3[1] << 8) | ((uint32_t)o3[2] << 16);
    }
    if (VPT == 2) ob = ((const uint16_t*)(stg + off_in_stage))[tp];
    if (VPT == 1) ob = stg[off_in_stage + tp];
}

// The update kernel.  VPT views per lane (4, or 1 for <= 128 views), uint8 or fp32 A, 8 or 26
// neighbours, R-voxel A-record ring, CL CTAs per task, KV voxels per step (1: exact sequential
// ICD within the SV; 2: voxel pairs from the same state); PROF adds per-phase cycle counters.
// T2: the theta2 pass -- theta2 = sum w A^2 (Alg1:6) is not precomputed yet: the view warps reduce
// it with theta1 in this iteration (which visits every voxel) and the delta warp stores it
// MB: the launch runs P.nbatch batches with grid barriers between them (cooperative launch);
// without it the batch loop compiles away (one batch per launch)
template <int VPT, bool U8, int NNB, int R, int CL, int KV, bool T2, bool PROF, bool MB>
__global__ void __launch_bounds__(max_threads(VPT), 1) k_svicd(const IcdParams P)
{
    extern __shared__ __align__(16) unsigned char smem[];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const int nvw = P.nvw / CL;            // view warps of this CTA (CL = 2: half of the task's)
    const uint32_t crank = CL == 1 ? 0u : cluster_rank();  // this CTA's rank in its cluster
    const bool is_view = warp < nvw, is_delta = warp == nvw, is_prior = warp == nvw + 1;
    const int vw = is_view ? warp : 0;
    const int V = P.V, M = P.M, S2 = P.S2, side = P.side;
    const int VA = P.A.VA;                 // record positions per voxel (all views)
    const int VAL = VA / CL;               // this CTA's record positions / SVB columns
    const int vbase = (int)crank * VAL;    // this CTA's first view
    constexpr int VS = svb_cols(VPT, CL);  // SVB row length (compile-time: row offsets are immediates)
    constexpr int RS = 2 * VS;             // float stride between consecutive e (or w) rows
    constexpr bool kNSL8 = VPT != 2;       // at most 8 view warps: only the first 8 slots are used
    const SmemLayout& L = P.lay;
    float* sb = (float*)(smem + L.sb_e);   // e row r at sb + r RS, w row r at sb + r RS + VS
    int* flags = (int*)(smem + L.flags);
    float* red = (float*)(smem + L.red);
    PriTerm* pri = (PriTerm*)(smem + L.pri);
    unsigned char* astage = smem + L.astage;
    float* stg_w = (float*)(smem + L.staging) + vw * 32 * kStg;
    int* s_task = (int*)(smem + L.misc);            // [b]: the task prepared in buffer b, [2 + b]: its kept voxels
    float* dslot = (float*)(smem + L.misc) + 4;     // [2 steps][2 voxels]: scale * delta of the step's voxels
    uint32_t* binfo = (uint32_t*)(smem + L.binfo);  // [2][VA], indexed by (global) view
    float* xs = (float*)(smem + L.cx);               // CL = 2: [2 steps][2 quantities][2 ranks] partial sums
    uint64_t* xbar = (uint64_t*)(smem + L.cx + 32);  // CL = 2: [2 steps] the peer's partials arrived
    uint64_t* tbar = xbar + 2;                       // CL = 2: [2 buffers] rank 0's task id arrived
    const int TW = side + 2;
    const int zc = (NNB == 26) ? 1 : 0;  // centre slice of the x tile
    const int ntile = (NNB == 26 ? 3 : 1) * TW * TW;  // x tile entries
    const size_t plane = (size_t)P.nx * P.ny;
    const int nab = (nvw + 1) * 32;      // barrier A: view warps + the delta warp
    const int nb2 = (nvw + 1) * 32;      // barrier B: view warps + the delta warp

    for (int i = threadIdx.x; i < 2 * 2 * 2 * kNSL; i += blockDim.x) red[i] = 0.f;  // slots >= nvw stay 0
    // the neighbourhood (reading R2) as shared-memory tables [dx | dy | dz | weight bits][32]: a
    // by-value kernel parameter indexed by a run-time value would be copied to local memory
    int* nbt = (int*)(smem + L.mbar);
    for (int i = threadIdx.x; i < 32; i += blockDim.x) {
        const bool ok = i < P.pc.nnb;
        nbt[i] = ok ? P.pc.dx[i] : 0;
        nbt[32 + i] = ok ? P.pc.dy[i] : 0;
        nbt[64 + i] = ok ? P.pc.dz[i] : 0;
        nbt[96 + i] = ok ? __float_as_int(P.pc.b[i]) : 0;
        nbt[128 + i] = ok ? (P.pc.dz[i] * (side + 2) + P.pc.dy[i]) * (side + 2) + P.pc.dx[i] : 0;
    }
    if (CL == 2 && threadIdx.x == 0) {
        for (int i = 0; i < 4; ++i) mbar_init(xbar + i, 1);  // one arrival: the peer's
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    if (CL == 2) cluster_sync_all();  // peer mbarriers initialised before any remote arrival
    uint32_t nfetch[2] = {0u, 0u};    // CL = 2: task ids received per buffer (tbar phases)
    // SVB rows outside a visit's band are never packed: start them finite (zero)
    for (int i = threadIdx.x; i < (L.xt - L.sb_e) / 16; i += blockDim.x)
        ((float4*)(smem + L.sb_e))[i] = make_float4(0.f, 0.f, 0.f, 0.f);
    // per-thread view ownership: view warp w, lane l owns views (w*VPT + t)*32 + l
    int kv[VPT];
#pragma unroll
    for (int t = 0; t < VPT; ++t) kv[t] = (vw * VPT + t) * 32 + lane;  // local SVB column
    uint32_t gseq = 0;  // running voxel sequence number of this CTA: A stage = gseq % R
    // prior-warp lane r owns neighbour r: offsets and weights in registers
    NbrOne nb;
    nb.dx = nbt[lane];
    nb.dy = nbt[32 + lane];
    nb.dz = nbt[64 + lane];
    nb.w = __int_as_float(nbt[96 + lane]);
    nb.dt = nbt[128 + lane];

    // this launch's batch: flat tasks [start, end) of the phase list (sched.cu k_flatten), pulled
    // one at a time by the persistent CTAs (dynamic distribution, Alg3:4 / T3); with the zero-skip
    // pre-filter (P.keep), tasks whose whole tile is zero are accounted as skipped visits here
    int tstart = P.brange[0], tend = P.brange[1];
    int* fetchp = P.fetch;
    auto fetch_task = [&]() {
        int q = tstart + atomicAdd(fetchp, 1);
        while (P.keep && q < tend && !P.keep[q]) {
            const int tkq = P.flat[q];
            const int zq = tkq >> 14, svq = tkq & 16383;
            const int twq = min(side, P.nx - (svq % P.nsvx) * side), thq = min(side, P.ny - (svq / P.nsvx) * side);
            P.sv_amount[(size_t)zq * P.nsv + svq] = 0.f;
            atomicAdd(P.counters + 1, (unsigned long long)(twq * thq));
            atomicAdd(P.counters + 2, 1ull);
            atomicAdd(P.counters + 3, 1ull);
            q = tstart + atomicAdd(fetchp, 1);
        }
        return q;
    };
    // ---- task preparation.  A task's inputs are stable during a phase (its own voxels are only
    //      updated by its owner, its ring belongs to other colours, its +-1 slices to the other z
    //      parity), so they are gathered early: while the current task is packed, the delta warp
    //      fetches the next task and copies its x tile (+1 halo ring, +-1 slice in 3-D; zeros
    //      off the image), the slots' scales and theta2 and its band start / width into shared
    //      memory with cp.async; during the current task's write-back the delta and prior warps
    //      (64 threads, named barrier kBarP) evaluate its zero-skip predicate (reading R9:
    //      slot kept iff valid and (skip inactive or x_j or a neighbour is non-zero) -- the tile
    //      holds zeros outside the volume), build its visiting order (one of NPERM host-drawn
    //      random permutations of the tile chosen per (seed, iteration, slice, SV) visit, raster
    //      order in deterministic mode, compacted with a ballot), stage the ordered scales and
    //      theta2 and its band info (+ an L2 warm-up of its band rows).  A task whose every voxel
    //      is skipped is accounted and replaced by the next one (synchronously).
    const int rt = threadIdx.x - nvw * 32;  // thread index among the delta and prior warps
    float* rscale = (float*)(smem + L.rscale);
    float* rth2 = (float*)(smem + L.rth2);
    int* rbs = (int*)(smem + L.rbs);
    unsigned char* rbw = smem + L.rbw;
    // delta warp: fetch the next task into s_task[b] and start copying its inputs into buffer b
    auto fetch_and_copy = [&](int b) {
        int qn = 0;
        if (crank == 0) {
            if (lane == 0) {
                qn = fetch_task();
                s_task[b] = qn;
                if (CL == 2) {  // rank 1 takes the same task
                    st_peer_u32(peer_addr(s_task + b, 1), (uint32_t)qn);
                    mbar_arrive_peer(peer_addr(tbar + b, 1));
                }
            }
        } else {
            if (lane == 0) mbar_wait_cluster(tbar + b, nfetch[b] & 1u);
            __syncwarp();
            qn = s_task[b];
        }
        ++nfetch[b];
        qn = __shfl_sync(kFull, qn, 0);
        if (qn < tend) {
            const int tkn = P.flat[qn];
            const int z = tkn >> 14, sv = tkn & 16383;
            const int gx0 = (sv % P.nsvx) * side, gy0 = (sv / P.nsvx) * side;
            float* xb = (float*)(smem + L.xt) + b * ntile;
            for (int i = lane; i < ntile; i += 32) {
                const int tz = i / (TW * TW), r = i % (TW * TW), ty = r / TW, tx = r % TW;
                const int gx = gx0 - 1 + tx, gy = gy0 - 1 + ty;
                const int zs = (NNB == 26) ? z + tz : z + 1;  // storage slice (halo at 0, nz+1)
                const bool inb = gx >= 0 && gx < P.nx && gy >= 0 && gy < P.ny;
                const int cx = min(max(gx, 0), P.nx - 1), cy = min(max(gy, 0), P.ny - 1);
                cp_async4_zfill(xb + i, P.x + (size_t)min(zs, P.nz_local + 1) * plane + (size_t)cy * P.nx + cx, inb);
            }
            const size_t arec = (size_t)sv * S2;
            for (int i = lane; i < S2; i += 32) {
                cp_async4(rscale + i, P.A.scale + arec + i);
                cp_async4(rth2 + i, P.theta2 + ((size_t)z * P.nsv + sv) * S2 + i);
            }
            for (int k = lane; k < V; k += 32) cp_async4(rbs + k, P.A.band_start + (size_t)sv * V + k);
            for (int k = 4 * lane; k < V; k += 128) {  // band widths as 4-byte words (V % 4 == 0)
                if ((V & 3) == 0) cp_async4(rbw + k, P.A.band_width + (size_t)sv * V + k);
            }
        }
        cp_async_commit();
    };
    // delta + prior warps: complete the preparation of the task in buffer b (copies issued by
    // fetch_and_copy); returns with s_task[b] >= tend or s_task[2 + b] > 0 kept voxels
    auto finish_prepare = [&](int b) {
        float* xb = (float*)(smem + L.xt) + b * ntile;
        int* listb = (int*)(smem + L.list) + b * S2;
        int* tofb = (int*)(smem + L.tof) + b * S2;
        for (;;) {
            if (is_delta) cp_async_wait<0>();
            bar_sync(kBarP, 64);
            const int qn = s_task[b];
            if (qn >= tend) return;
            const int tkn = P.flat[qn];
            const int z = tkn >> 14, sv = tkn & 16383, zg = P.z_offset + z;
            const int gx0 = (sv % P.nsvx) * side, gy0 = (sv / P.nsvx) * side;
            const int tw = min(side, P.nx - gx0), th = min(side, P.ny - gy0);
            for (int v0 = rt; v0 < S2; v0 += 64) {
                const int lx = v0 % side, ly = v0 / side;
                int keep = lx < tw && ly < th;
                if (keep && P.zero_skip_active) {
                    const float* c = xb + (zc * TW + ly + 1) * TW + lx + 1;
                    float acc = fabsf(c[0]);
#pragma unroll
                    for (int r = 0; r < NNB; ++r) acc += fabsf(c[nbt[128 + r]]);
                    keep = acc != 0.f;
                }
                flags[v0] = keep;
            }
            bar_sync(kBarP, 64);
            if (is_prior) {
                const uint64_t h = mix64(P.seed ^ mix64(((uint64_t)P.iter << 40) ^ ((uint64_t)zg << 20) ^ (uint64_t)sv));
                const uint8_t* perm = P.perm + (size_t)(h % (uint64_t)P.nperm) * S2;
                int n = 0;
                for (int base = 0; base < S2; base += 32) {
                    const int i = base + lane;
                    const int v = i < S2 ? (P.deterministic ? i : (int)perm[i]) : 0;
                    const bool k = i < S2 && flags[v];
                    const unsigned m = __ballot_sync(kFull, k);
                    if (k) {
                        const int p = n + __popc(m & ((1u << lane) - 1));
                        listb[p] = v;
                        tofb[p] = ((v / side) << 8) | (v % side);  // packed (ly, lx): no div in the loop
                    }
                    n += __popc(m);
                }
                if (lane == 0) {
                    s_task[2 + b] = n;
                    if (n == 0 && crank == 0) {  // the whole SV is zero-skipped: account for it
                        P.sv_amount[(size_t)z * P.nsv + sv] = 0.f;
                        atomicAdd(P.counters + 1, (unsigned long long)(tw * th));
                        atomicAdd(P.counters + 2, 1ull);
                        atomicAdd(P.counters + 3, 1ull);
                    }
                }
                __syncwarp();
                float* vsb = (float*)(smem + L.vscale) + b * S2;
                float* vtb = (float*)(smem + L.vth2) + b * S2;
                for (int i = lane; i < n; i += 32) {
                    const int v = listb[i];
                    vsb[i] = rscale[v];
                    vtb[i] = rth2[v];
                }
                if (n > 0) {
                    // band info (row offset << 6 | width) and an L2 warm-up of the band rows
                    uint32_t* dst = binfo + b * VA;
                    const float* wz = P.w + (size_t)z * V * M;
                    const float* ez = P.e + (size_t)z * V * M;
                    for (int k = lane; k < V; k += 32) {
                        const int wd = (V & 3) == 0 ? rbw[k] : P.A.band_width[(size_t)sv * V + k];
                        const int r = k * M + rbs[k], r1 = r + max(wd, 1) - 1;
                        dst[k] = ((uint32_t)r << 6) | (uint32_t)wd;
                        asm volatile("prefetch.global.L2 [%0];" ::"l"(wz + r));
                        asm volatile("prefetch.global.L2 [%0];" ::"l"(wz + r1));
                        asm volatile("prefetch.global.L2 [%0];" ::"l"(ez + r));
                        asm volatile("prefetch.global.L2 [%0];" ::"l"(ez + r1));
                    }
                }
            }
            bar_sync(kBarP, 64);
            if (s_task[2 + b] > 0) return;
            if (is_delta) fetch_and_copy(b);  // fully skipped: the next task, synchronously
        }
    };
    // the launch's batches (Alg3:24-27: each batch sees the previous one's write-backs): a grid
    // barrier between two (the launch is cooperative when nbatch > 1, so every CTA is resident).
    // Task inputs other than e are stable within a phase, so only e needs the barrier's ordering
    const int nbatch = MB ? P.nbatch : 1;
    for (int bt = 0; bt < nbatch; ++bt) {
    if (MB) {
        tstart = P.brange[bt];
        tend = P.brange[bt + 1];
        fetchp = P.fetch + bt;
    }
    int cb = 0;  // buffer of the current task (binfo, x tile, order, scales)
    if (is_delta) fetch_and_copy(0);
    if (!is_view) finish_prepare(0);
    __syncthreads();
    int q = s_task[0];
    for (; q < tend; q = s_task[cb ^ 1], cb ^= 1) {
        const int tk = P.flat[q];
        const int z = tk >> 14, sv = tk & 16383;  // local slice, SV
        const int zg = P.z_offset + z;            // global slice
        const int gx0 = (sv % P.nsvx) * side, gy0 = (sv / P.nsvx) * side;
        const int tw = min(side, P.nx - gx0), th = min(side, P.ny - gy0);
        const int tb = cb;
        float* xt = (float*)(smem + L.xt) + cb * ntile;
        const int* list = (const int*)(smem + L.list) + cb * S2;
        const int* tof = (const int*)(smem + L.tof) + cb * S2;
        const float* vscale = (const float*)(smem + L.vscale) + cb * S2;
        const float* vth2 = (const float*)(smem + L.vth2) + cb * S2;
        const int nactv = s_task[2 + cb];
        long long tp0 = 0, tp1 = 0, tp2 = 0, tp3 = 0;
        if (PROF && threadIdx.x == 0) tp0 = clock64();
        const size_t arec = (size_t)sv * S2;  // first A record of this SV
        constexpr int CB = U8 ? 4 : 16;       // record bytes per view position
        const int tpm = vw * 32 + lane;
        const unsigned char* g_code = (const unsigned char*)(U8 ? (const void*)P.A.codes : (const void*)P.A.vals) +
                                      ((size_t)arec * VA + vbase + tpm * VPT) * CB;
        const unsigned char* g_off = P.A.off + (size_t)arec * VA + vbase + tpm * VPT;
        // view thread: asynchronous copy of its own slice of voxel j's record into ring stage stg,
        // one commit group per voxel (empty past the visit's end)
        auto copy_record_to = [&](int j, int stg, int v) {
            if (j < nactv) {
                unsigned char* st = astage + stg * L.stage_bytes;
                const unsigned char* gc = g_code + (size_t)v * (VA * CB);
                if (U8) {
                    if (VPT == 4)
                        cp_async16(st + tpm * 16, gc);
                    else if (VPT == 2)
                        cp_async8(st + tpm * 8, gc);
                    else
#pragma unroll
                        for (int t = 0; t < VPT; ++t) cp_async4(st + (tpm * VPT + t) * 4, gc + t * 4);
                } else {
#pragma unroll
                    for (int t = 0; t < VPT; ++t) cp_async16(st + (tpm * VPT + t) * 16, gc + t * 16);
                }
                if (VPT == 3) {  // offsets: 3 bytes per thread, 4 threads' 12 bytes as 3 words
                    if ((tpm & 3) == 0)
#pragma unroll
                        for (int t = 0; t < 3; ++t) cp_async4(st + L.off_in_stage + tpm * 3 + 4 * t, g_off + (size_t)v * VA + 4 * t);
                } else if ((tpm & (4 / VPT - 1)) == 0) {  // offsets: VPT bytes per thread, as 4-byte words
                    cp_async4(st + L.off_in_stage + tpm * VPT, g_off + (size_t)v * VA);
                }
            }
            cp_async_commit();
        };
        const int sbase = (int)(gseq % (uint32_t)R);  // ring stage of this visit's voxel 0
        const int cslot = (zc * TW + 1) * TW + 1;     // tile index of local (0,0)
        // the first voxel's surrogate terms (prior warp) and the next task's input copies (delta
        // warp) while the view warps pack
        if (is_prior) {
            if (KV == 1) {
                prior_one<1>(tof, 0, -1, -1, xt, cslot, TW, gx0, gy0, zg, P, nb, lane, pri + 2 * (gseq & 1));
            } else {  // pair 0: both from the same state
                prior_one<2>(tof, 0, -1, -1, xt, cslot, TW, gx0, gy0, zg, P, nb, lane, pri);
                if (nactv > 1) prior_one<2>(tof, 1, -1, -1, xt, cslot, TW, gx0, gy0, zg, P, nb, lane, pri + 1);
            }
            __syncwarp();
        } else if (is_delta) {
            fetch_and_copy(cb ^ 1);
        }
        if (PROF && threadIdx.x == 0) tp1 = clock64();

        // ---- 4. view warps: SVB pack (coalesced band-row windows transposed through staging
        //         tiles); e_init rows go to this CTA's L2-resident scratch tile for the write-back
        const int nwin = P.nwin;  // 32-float windows per band row (2: bands of 30..61 rows)
        float* scr = P.scratch + (size_t)blockIdx.x * (size_t)nwin * VS * 32;
        const int ntw = tile_warps(VAL);
        if (is_view && vw < ntw) {
            const float* wz = P.w + (size_t)z * V * M;
            float* ez = P.e + (size_t)z * V * M;
            // Each band row is read as the 16-byte-aligned 32-float window(s) that contain it (the
            // slice base is 16-byte aligned, V*M % 4 == 0): 8 lanes x float4 per row, 4 rows per
            // LDG.128; the window goes through the warp's staging tile and band column
            // c = p - s_k lands in sb row c, column k (bank k)
            const int sub = lane >> 3, ch = lane & 7;  // row-in-quad and float4 chunk of this lane
            int wq = 0;                                // window of the band rows (0, 1)
            auto issue = [&](int t, bool isw, float4 (&v4)[8]) {
                const int kk = vbase + (vw * kTileW + t) * 32 + lane;  // global view
                const uint32_t bi = kk < V ? binfo[tb * VA + kk] : 0u;
                const int rot = (int)(bi >> 6);
#pragma unroll
                for (int m = 0; m < 8; ++m) {
                    const int oi = __shfl_sync(kFull, rot, 4 * m + sub);
                    // unconditional loads: the whole aligned window is read (padded views read the
                    // slice start; the sinogram allocations carry 64 floats of tail padding)
                    const size_t a4 = (size_t)(oi - (oi & 3)) + 32 * wq + 4 * ch;
                    v4[m] = isw ? __ldg((const float4*)(wz + a4)) : __ldcg((const float4*)(ez + a4));
                }
            };
            auto finish = [&](int t, bool isw, const float4 (&v4)[8]) {
                const int k0 = (vw * kTileW + t) * 32;  // local column of the tile
                const uint32_t bi = vbase + k0 + lane < V ? binfo[tb * VA + vbase + k0 + lane] : 0u;
                const int kk = k0 + lane;
                const int bwt = (int)(bi & 63u), sk = (int)(bi >> 6) & 3;
                // the band's positions in this window
                const uint32_t bmask = (uint32_t)((((1ull << bwt) - 1ull) << sk) >> (32 * wq));
                if (!isw) {
#pragma unroll
                    for (int m = 0; m < 8; ++m)
                        __stcg((float4*)(scr + ((size_t)wq * VS + k0 + 4 * m + sub) * 32 + 4 * ch), v4[m]);
                }
                float* d = sb + (isw ? VS : 0) + kk + (32 * wq - sk) * RS;  // + p RS = band row 32 wq + p - sk
#pragma unroll
                for (int m = 0; m < 8; ++m) *(float4*)(stg_w + (4 * m + sub) * kStg + 4 * ch) = v4[m];
                __syncwarp();
#pragma unroll
                for (int q4 = 0; q4 < 8; ++q4) {
                    const float4 r = lds128(stg_w + lane * kStg + 4 * q4);
                    const float rv[4] = {r.x, r.y, r.z, r.w};
#pragma unroll
                    for (int j = 0; j < 4; ++j)
                        if (bmask & (1u << (4 * q4 + j))) d[(4 * q4 + j) * RS] = rv[j];
                }
                __syncwarp();
            };
            for (wq = 0; wq < nwin; ++wq) {
                float4 wa4[2][8], ea4[2][8];
                issue(0, true, wa4[0]);
                issue(0, false, ea4[0]);
#pragma unroll
                for (int t = 0; t < kTileW; ++t) {
                    if (t + 1 < kTileW) {
                        issue(t + 1, true, wa4[(t + 1) & 1]);
                        issue(t + 1, false, ea4[(t + 1) & 1]);
                    }
                    finish(t, true, wa4[t & 1]);
                    finish(t, false, ea4[t & 1]);
                }
            }
        }
        __syncthreads();
        if (PROF && threadIdx.x == 0) tp2 = clock64();

        // ---- 5. the voxel loop, exactly sequential ICD one voxel per step: the view warps gather
        //         theta1's partials of voxel i from e (after voxel i - 1's scatter) and arrive on A;
        //         the delta warp (A also waits for the prior warp's terms of i) writes voxel i - 1's
        //         new value into the x tile (releasing the prior warp, X, to compute voxel i + 1's
        //         terms), corrects i's terms if i - 1 is its neighbour, derives delta_i and
        //         publishes it (B); meanwhile the view warps prepare voxel i + 1 (A record, w A);
        //         after B they scatter voxel i into their own views.
        float amount = 0.f;
        const uint32_t g0 = gseq;  // step buffers alternate with the running voxel number
        if (is_view) {
            const int tp = tpm;
            constexpr int CW = U8 ? 1 : 4;  // record words per view
            // per-voxel state of a view thread for its VPT views: the band offsets (packed bytes),
            // the float index of each view's first row in sb, the dequantised A and w*A
            struct VoxState {
                int p[VPT];
                float2 f[VPT][2], wf[VPT][2];
                int sj;  // ring stage of the voxel's record
            };
            auto avals = [&](const uint32_t (&c)[CW], float2 (&f)[2]) {
                if (U8) {
                    f[0] = dq2(c[0], 0);
                    f[1] = dq2(c[0], 2);
                } else {
                    f[0] = make_float2(__uint_as_float(c[0]), __uint_as_float(c[CW > 1 ? 1 : 0]));
                    f[1] = make_float2(__uint_as_float(c[CW > 2 ? 2 : 0]), __uint_as_float(c[CW > 3 ? 3 : 0]));
                }
            };
            // voxel j of the visiting order -> vs (e-independent: record, offsets, w A)
            auto prep = [&](VoxState& vs) {
                cp_async_wait<R - 1>();      // this thread's copy of the voxel's record has landed
                if (VPT != 4) __syncwarp();  // offset words copied by another lane of the warp
                uint32_t c[VPT][CW], ow;
                load_words<VPT, CW>(astage + vs.sj * L.stage_bytes, L.off_in_stage, tp, c, ow);
#pragma unroll
                for (int t = 0; t < VPT; ++t) {
                    avals(c[t], vs.f[t]);
                    vs.p[t] = (int)((ow >> (8 * t)) & 255u) * RS + kv[t];
                    const float* pw = sb + VS + vs.p[t];
                    vs.wf[t][0] = __fmul2_rn(make_float2(pw[0], pw[RS]), vs.f[t][0]);
                    vs.wf[t][1] = __fmul2_rn(make_float2(pw[2 * RS], pw[3 * RS]), vs.f[t][1]);
                }
            };
            // refill the stage voxel j's record used with the record R voxels ahead (one commit
            // group per voxel, empty past the visit's end, keeps the wait counts fixed)
            auto refill = [&](int j, int sj) {
                if (VPT != 4) __syncwarp();  // lanes read offset words another lane refills
                copy_record_to(j + R, sj, j + R < nactv ? list[j + R] : 0);
            };
            auto step = [&](int idx, VoxState& cur, VoxState& nxt) {
                const uint32_t sn = (g0 + (uint32_t)idx) & 1u;
                float2 ev[VPT][2];
                {
                    float2 acc[2] = {make_float2(0.f, 0.f), make_float2(0.f, 0.f)};
                    float2 acc2 = make_float2(0.f, 0.f);  // T2: w A^2 (unscaled codes)
#pragma unroll
                    for (int t = 0; t < VPT; ++t) {
                        const float* pe = sb + cur.p[t];
                        ev[t][0] = make_float2(pe[0], pe[RS]);
                        ev[t][1] = make_float2(pe[2 * RS], pe[3 * RS]);
                        acc[t & 1] = __ffma2_rn(cur.wf[t][0], ev[t][0], acc[t & 1]);
                        acc[t & 1] = __ffma2_rn(cur.wf[t][1], ev[t][1], acc[t & 1]);
                        if (T2) {
                            acc2 = __ffma2_rn(cur.wf[t][0], cur.f[t][0], acc2);
                            acc2 = __ffma2_rn(cur.wf[t][1], cur.f[t][1], acc2);
                        }
                    }
                    const float2 ac = __fadd2_rn(acc[0], acc[1]);
                    float g = ac.x + ac.y, g2 = acc2.x + acc2.y;
#pragma unroll
                    for (int o = 16; o > 0; o >>= 1) {
                        g += __shfl_xor_sync(kFull, g, o);
                        if (T2) g2 += __shfl_xor_sync(kFull, g2, o);
                    }
                    if (lane == 0) {
                        red[sn * 4 * kNSL + vw] = g;
                        if (T2) red[sn * 4 * kNSL + kNSL + vw] = g2;
                    }
                }
                bar_arrive(kBarA, nab);
                // meanwhile: the next voxel's e-independent state, then refill its stage
                nxt.sj = cur.sj + 1 == R ? 0 : cur.sj + 1;
                if (idx + 1 < nactv) prep(nxt);
                refill(idx + 1, nxt.sj);
                bar_sync(kBarB, nb2);
                // Alg1:9-11 on this thread's views
                const float sd = dslot[2 * sn];
                if (sd != 0.f) {
                    const float2 nd = make_float2(-sd, -sd);
#pragma unroll
                    for (int t = 0; t < VPT; ++t) {
                        float* pe = sb + cur.p[t];
                        const float2 a0 = __ffma2_rn(cur.f[t][0], nd, ev[t][0]);
                        const float2 a1 = __ffma2_rn(cur.f[t][1], nd, ev[t][1]);
                        pe[0] = a0.x;
                        pe[RS] = a0.y;
                        pe[2 * RS] = a1.x;
                        pe[3 * RS] = a1.y;
                    }
                }
            };
            // the first R records (the ring region held the pack's staging tiles until the barrier)
            for (int i = 0; i < R; ++i) copy_record_to(i, (sbase + i) % R, i < nactv ? list[i] : 0);
            if constexpr (KV == 1) {
                VoxState st0, st1;
                st0.sj = sbase;
                prep(st0);
                refill(0, sbase);
                for (int idx = 0; idx < nactv; idx += 2) {
                    step(idx, st0, st1);
                    if (idx + 1 < nactv) step(idx + 1, st1, st0);
                }
            } else {
                // ---- voxel pairs (intra-SV parallelism): step s updates voxels
                //      2s and 2s + 1 from the same e and x (Jacobi within the pair); the second
                //      voxel's scatter re-reads the rows the first one's may have changed
                auto prep_j = [&](int j, VoxState& vs) {
                    vs.sj = (sbase + j) % R;
                    if (j < nactv) {
                        prep(vs);
                    } else {  // past the visit's end: a null voxel (no loads, nothing scattered)
#pragma unroll
                        for (int t = 0; t < VPT; ++t) {
                            vs.p[t] = kv[t];
                            vs.f[t][0] = vs.f[t][1] = vs.wf[t][0] = vs.wf[t][1] = make_float2(0.f, 0.f);
                        }
                    }
                    refill(j, vs.sj);
                };
                auto pstep = [&](int s2, VoxState& ca, VoxState& cb, VoxState& na, VoxState& nb) {
                    const int sn = s2 & 1;
                    float2 eva[VPT][2], evb[VPT][2];
                    {
                        float2 aa = make_float2(0.f, 0.f), ab = make_float2(0.f, 0.f);
                        float2 qa = make_float2(0.f, 0.f), qb = make_float2(0.f, 0.f);  // T2
#pragma unroll
                        for (int t = 0; t < VPT; ++t) {
                            const float* pa = sb + ca.p[t];
                            const float* pb = sb + cb.p[t];
                            eva[t][0] = make_float2(pa[0], pa[RS]);
                            eva[t][1] = make_float2(pa[2 * RS], pa[3 * RS]);
                            evb[t][0] = make_float2(pb[0], pb[RS]);
                            evb[t][1] = make_float2(pb[2 * RS], pb[3 * RS]);
                            aa = __ffma2_rn(ca.wf[t][0], eva[t][0], aa);
                            ab = __ffma2_rn(cb.wf[t][0], evb[t][0], ab);
                            aa = __ffma2_rn(ca.wf[t][1], eva[t][1], aa);
                            ab = __ffma2_rn(cb.wf[t][1], evb[t][1], ab);
                            if (T2) {
                                qa = __ffma2_rn(ca.wf[t][0], ca.f[t][0], qa);
                                qb = __ffma2_rn(cb.wf[t][0], cb.f[t][0], qb);
                                qa = __ffma2_rn(ca.wf[t][1], ca.f[t][1], qa);
                                qb = __ffma2_rn(cb.wf[t][1], cb.f[t][1], qb);
                            }
                        }
                        float ga = aa.x + aa.y, gb = ab.x + ab.y, g2a = qa.x + qa.y, g2b = qb.x + qb.y;
#pragma unroll
                        for (int o = 16; o > 0; o >>= 1) {
                            ga += __shfl_xor_sync(kFull, ga, o);
                            gb += __shfl_xor_sync(kFull, gb, o);
                            if (T2) {
                                g2a += __shfl_xor_sync(kFull, g2a, o);
                                g2b += __shfl_xor_sync(kFull, g2b, o);
                            }
                        }
                        if (lane == 0) {  // red[step][voxel][theta1, theta2][slot]
                            red[(4 * sn + 0) * kNSL + vw] = ga;
                            red[(4 * sn + 2) * kNSL + vw] = gb;
                            if (T2) {
                                red[(4 * sn + 1) * kNSL + vw] = g2a;
                                red[(4 * sn + 3) * kNSL + vw] = g2b;
                            }
                        }
                    }
                    bar_arrive(kBarA, nab);
                    // meanwhile: the next pair's e-independent state
                    prep_j(2 * s2 + 2, na);
                    prep_j(2 * s2 + 3, nb);
                    bar_sync(kBarB, nb2);
                    // Alg1:9-11 on this thread's views: voxel a from its gathered values, then
                    // voxel b on the current e (a's scatter may have changed rows b reads)
                    const float sda = dslot[2 * sn], sdb = dslot[2 * sn + 1];
                    if (sda != 0.f) {
                        const float2 nd = make_float2(-sda, -sda);
#pragma unroll
                        for (int t = 0; t < VPT; ++t) {
                            float* pe = sb + ca.p[t];
                            const float2 a0 = __ffma2_rn(ca.f[t][0], nd, eva[t][0]);
                            const float2 a1 = __ffma2_rn(ca.f[t][1], nd, eva[t][1]);
                            pe[0] = a0.x;
                            pe[RS] = a0.y;
                            pe[2 * RS] = a1.x;
                            pe[3 * RS] = a1.y;
                        }
                    }
                    if (sdb != 0.f) {
                        const float2 nd = make_float2(-sdb, -sdb);
#pragma unroll
                        for (int t = 0; t < VPT; ++t) {
                            float* pe = sb + cb.p[t];
                            if (sda != 0.f && abs(cb.p[t] - ca.p[t]) < 4 * RS) {  // rows overlap
                                evb[t][0] = make_float2(pe[0], pe[RS]);
                                evb[t][1] = make_float2(pe[2 * RS], pe[3 * RS]);
                            }
                            const float2 b0 = __ffma2_rn(cb.f[t][0], nd, evb[t][0]);
                            const float2 b1 = __ffma2_rn(cb.f[t][1], nd, evb[t][1]);
                            pe[0] = b0.x;
                            pe[RS] = b0.y;
                            pe[2 * RS] = b1.x;
                            pe[3 * RS] = b1.y;
                        }
                    }
                };
                VoxState a0, b0, a1, b1;
                prep_j(0, a0);
                prep_j(1, b0);
                const int nsteps = (nactv + 1) >> 1;
                for (int s2 = 0; s2 < nsteps; s2 += 2) {
                    pstep(s2, a0, b0, a1, b1);
                    if (s2 + 1 < nsteps) pstep(s2 + 1, a1, b1, a0, b0);
                }
            }
        } else if (is_delta) {
          if constexpr (KV == 2) {
            // ---- delta warp, voxel pairs: as below for both voxels of a step, from the same state
            float upa = 0.f, vpa = 0.f, upb = 0.f, vpb = 0.f;  // the previous pair's new / old values
            const int nsteps = (nactv + 1) >> 1;
            auto put_x = [&](int i, float u) {
                const int tu = tof[i];
                xt[cslot + (tu >> 8) * TW + (tu & 255)] = u;
            };
            // voxel i's prior part with the previous pair's new values (terms reported by the prior warp)
            auto prior_part = [&](const PriTerm& pp, float& ps, float& psx) {
                ps = pp.s;
                psx = pp.sx;
                if (pp.bwu0 != 0.f) {
                    const float bn = pp.bwu0 * phi_f(P.pc, pp.v - upa);
                    ps += bn - pp.btu0;
                    psx += bn * upa - pp.btu0 * vpa;
                }
                if (pp.bwu1 != 0.f) {
                    const float bn = pp.bwu1 * phi_f(P.pc, pp.v - upb);
                    ps += bn - pp.btu1;
                    psx += bn * upb - pp.btu1 * vpb;
                }
            };
            for (int s2 = 0; s2 < nsteps; ++s2) {
                const int sn = s2 & 1;
                const int ia = 2 * s2, ib = ia + 1;
                const bool hb = ib < nactv;
                bar_sync(kBarT, 64);
                if (s2 > 0 && lane == 0) {  // the previous pair's new values (a full pair)
                    put_x(ia - 2, upa);
                    put_x(ia - 1, upb);
                }
                bar_arrive(kBarX, 64);
                const PriTerm pa = pri[2 * sn], pb = pri[2 * sn + 1];
                float psa, psxa, psb = 0.f, psxb = 0.f;
                prior_part(pa, psa, psxa);
                if (hb) prior_part(pb, psb, psxb);
                const float sca = vscale[ia], scb = hb ? vscale[ib] : 0.f;
                float t2a = T2 ? 0.f : vth2[ia], t2b = (T2 || !hb) ? 0.f : vth2[ib];
                float dena = t2a + 2.f * psa, denb = t2b + 2.f * psb;
                float c1a = t2a * pa.v + 2.f * psxa, c1b = t2b * pb.v + 2.f * psxb;
                float ra = dena > 0.f ? __fdividef(1.f, dena) : 0.f, rb = denb > 0.f ? __fdividef(1.f, denb) : 0.f;
                bar_sync(kBarA, nab);
                const float Sa = slot_sum<kNSL8>(red + (4 * sn + 0) * kNSL);
                const float Sb = slot_sum<kNSL8>(red + (4 * sn + 2) * kNSL);
                if (T2) {  // theta2 of both voxels, stored for the later iterations
                    const float wa = slot_sum<kNSL8>(red + (4 * sn + 1) * kNSL);
                    const float wb = slot_sum<kNSL8>(red + (4 * sn + 3) * kNSL);
                    t2a = U8 ? sca * sca * wa : wa;
                    t2b = U8 ? scb * scb * wb : wb;
                    dena = t2a + 2.f * psa;
                    denb = t2b + 2.f * psb;
                    c1a = t2a * pa.v + 2.f * psxa;
                    c1b = t2b * pb.v + 2.f * psxb;
                    ra = dena > 0.f ? __fdividef(1.f, dena) : 0.f;
                    rb = denb > 0.f ? __fdividef(1.f, denb) : 0.f;
                    if (lane == 0) {
                        float* th = P.theta2 + ((size_t)z * P.nsv + sv) * S2;
                        th[list[ia]] = t2a;
                        if (hb) th[list[ib]] = t2b;
                    }
                }
                // Alg1:5-8 for both voxels
                const float th1a = -sca * Sa, th1b = -scb * Sb;
                float ua = pa.v, ub = pb.v;
                if (dena > 0.f) ua = (c1a - th1a) * ra;
                if (denb > 0.f) ub = (c1b - th1b) * rb;
                if (P.pc.positivity) {
                    ua = fmaxf(ua, 0.f);
                    ub = fmaxf(ub, 0.f);
                }
                const float da = ua - pa.v, db = hb ? ub - pb.v : 0.f;
                if (lane == 0) {
                    dslot[2 * sn] = sca * da;
                    dslot[2 * sn + 1] = scb * db;
                }
                bar_arrive(kBarB, nb2);
                upa = ua;
                vpa = pa.v;
                upb = ub;
                vpb = pb.v;
                if (lane == 0) {
                    amount += fabsf(da) + fabsf(db);
                    if (P.dump) {
                        // test hook: both updates; the second carries bit 31 (computed from the
                        // same state as the record before it)
                        const int nrec = hb ? 2 : 1;
                        const unsigned long long slot = atomicAdd(P.dump_count, (unsigned long long)nrec);
                        for (int r = 0; r < nrec; ++r) {
                            const int tv = tof[ia + r];
                            const uint32_t vox = (uint32_t)(((size_t)z * P.ny + gy0 + (tv >> 8)) * P.nx + gx0 + (tv & 255)) |
                                                 (r ? 0x80000000u : 0u);
                            if (slot + r < (unsigned long long)P.dump_cap)
                                *(float4*)(P.dump + 4 * (slot + r)) =
                                    make_float4(__uint_as_float(vox), r ? th1b : th1a, r ? t2b : t2a, r ? db : da);
                        }
                    }
                }
            }
            if (lane == 0) {  // the last pair's new values
                const int ia = 2 * (nsteps - 1);
                put_x(ia, upa);
                if (ia + 1 < nactv) put_x(ia + 1, upb);
            }
            __syncwarp();
          } else {
            // ---- delta warp (every lane computes the same values; lane 0 publishes).  The prior
            //      side of the update (voxel i - 1's neighbour correction, the numerator's and the
            //      denominator's prior terms, the reciprocal) is done as soon as the prior warp's
            //      terms are in (T), before the view warps' partial sums (A): after A only
            //      theta1, one FMA and the clip remain on the chain
            float u_prev = 0.f, v_prev = 0.f;
            for (int idx = 0; idx < nactv; ++idx) {
                const uint32_t sn = (g0 + (uint32_t)idx) & 1u;
                bar_sync(kBarT, 64);
                if (idx > 0 && lane == 0) {  // voxel i - 1's new value, deferred until the prior
                    const int tu = tof[idx - 1];  // warp has computed voxel i's terms with the old one
                    xt[cslot + (tu >> 8) * TW + (tu & 255)] = u_prev;
                }
                bar_arrive(kBarX, 64);
                const PriTerm pp = pri[2 * sn];
                float ps = pp.s, psx = pp.sx;
                if (pp.bwu0 != 0.f) {  // voxel i - 1 is a neighbour: its term at its new value
                    const float bn = pp.bwu0 * phi_f(P.pc, pp.v - u_prev);
                    ps += bn - pp.btu0;
                    psx += bn * u_prev - pp.btu0 * v_prev;
                }
                const float scale = vscale[idx];
                float theta2 = T2 ? 0.f : vth2[idx];  // Alg1:6 (precomputed, or reduced below)
                float den = theta2 + 2.f * ps;
                float c1 = theta2 * pp.v + 2.f * psx;  // numerator without -theta1
                float rden = den > 0.f ? __fdividef(1.f, den) : 0.f;
                bar_sync(kBarA, nab);
                float S = slot_sum<kNSL8>(red + sn * 4 * kNSL);
                float Sw = T2 ? slot_sum<kNSL8>(red + sn * 4 * kNSL + kNSL) : 0.f;
                if (CL == 2) {
                    // this CTA's partial sums to both CTAs; the peer's arrive on xbar[sn] (its
                    // phase flips every second step); both add in rank order: identical bits
                    float* xq = xs + sn * 4;  // [theta1, theta2][rank]
                    if (lane == 0) {
                        xq[crank] = S;
                        st_peer_f32(peer_addr(xq + crank, crank ^ 1u), S);
                        if (T2) {
                            xq[2 + crank] = Sw;
                            st_peer_f32(peer_addr(xq + 2 + crank, crank ^ 1u), Sw);
                        }
                        mbar_arrive_peer(peer_addr(xbar + sn, crank ^ 1u));
                        mbar_wait_cluster(xbar + sn, ((g0 + (uint32_t)idx) >> 1) & 1u);
                    }
                    __syncwarp();
                    S = xq[0] + xq[1];
                    if (T2) Sw = xq[2] + xq[3];
                }
                if (T2) {  // theta2 of this voxel, stored for the later iterations
                    theta2 = U8 ? scale * scale * Sw : Sw;
                    den = theta2 + 2.f * ps;
                    c1 = theta2 * pp.v + 2.f * psx;
                    rden = den > 0.f ? __fdividef(1.f, den) : 0.f;
                    if (lane == 0 && crank == 0) P.theta2[((size_t)z * P.nsv + sv) * S2 + list[idx]] = theta2;
                }
                const float theta1 = -scale * S;  // Alg1:5
                float u = pp.v;
                if (den > 0.f) u = (c1 - theta1) * rden;
                if (P.pc.positivity) u = fmaxf(u, 0.f);
                const float d = u - pp.v;  // Alg1:7-8
                if (lane == 0) dslot[2 * sn] = scale * d;
                bar_arrive(kBarB, nb2);
                u_prev = u;
                v_prev = pp.v;
                if (lane == 0) {
                    amount += fabsf(d);
                    if (P.dump && crank == 0) {
                        // test hook (mbir_set_update_dump): the update's (voxel, theta1, theta2,
                        // delta) exactly as the delta chain used them
                        const unsigned long long slot = atomicAdd(P.dump_count, 1ull);
                        const int tv = tof[idx];
                        const uint32_t vox = (uint32_t)(((size_t)z * P.ny + gy0 + (tv >> 8)) * P.nx + gx0 + (tv & 255));
                        if (slot < (unsigned long long)P.dump_cap)
                            *(float4*)(P.dump + 4 * slot) = make_float4(__uint_as_float(vox), theta1, theta2, d);
                    }
                }
            }
            if (lane == 0) {  // the last voxel's new value
                const int tu = tof[nactv - 1];
                xt[cslot + (tu >> 8) * TW + (tu & 255)] = u_prev;
            }
            __syncwarp();
          }
        } else if (is_prior && KV == 2) {
            // ---- prior warp, voxel pairs: pair s + 1's terms (both with pair s's old values,
            //      reported for the correction) once pair s - 1's new values are in the tile (X)
            bar_arrive(kBarT, 64);  // pair 0's terms were computed during the pack
            const int nsteps = (nactv + 1) >> 1;
            for (int s2 = 0; s2 < nsteps; ++s2) {
                bar_sync(kBarX, 64);
                if (s2 + 1 < nsteps) {
                    const int ia = 2 * s2 + 2;
                    PriTerm* out = pri + 2 * ((s2 + 1) & 1);
                    prior_one<2>(tof, ia, ia - 2, ia - 1, xt, cslot, TW, gx0, gy0, zg, P, nb, lane, out);
                    if (ia + 1 < nactv)
                        prior_one<2>(tof, ia + 1, ia - 2, ia - 1, xt, cslot, TW, gx0, gy0, zg, P, nb, lane, out + 1);
                    __syncwarp();
                    bar_arrive(kBarT, 64);
                }
            }
        } else if (is_prior) {
            // ---- prior warp: voxel i + 1's terms once voxel i - 1's new value is in the tile (X);
            //      its arrival on A completes voxel i + 1's inputs
            bar_arrive(kBarT, 64);  // voxel 0's terms were computed during the pack
            for (int idx = 0; idx < nactv; ++idx) {
                bar_sync(kBarX, 64);
                if (idx + 1 < nactv) {
                    prior_one<1>(tof, idx + 1, idx, -1, xt, cslot, TW, gx0, gy0, zg, P, nb, lane,
                                 pri + 2 * ((g0 + (uint32_t)idx + 1) & 1));
                    __syncwarp();
                    bar_arrive(kBarT, 64);
                }
            }
        }
        gseq += nactv;
        if (PROF && threadIdx.x == 0) tp3 = clock64();
        __syncthreads();

        // ---- 6. write-back: delta e of the band, atomically, and the SV's voxels
        if (is_view && vw < ntw) {
            float* ez = P.e + (size_t)z * V * M;
            const int sub = lane >> 3, ch = lane & 7;
            for (int wq = 0; wq < nwin; ++wq) {
            auto ld_init = [&](int t, float4 (&s4)[8]) {
                const int k0 = (vw * kTileW + t) * 32;
#pragma unroll
                for (int m = 0; m < 8; ++m)
                    s4[m] = __ldcg((const float4*)(scr + ((size_t)wq * VS + k0 + 4 * m + sub) * 32 + 4 * ch));
            };
            float4 s4b[2][8];
            ld_init(0, s4b[0]);
#pragma unroll
            for (int t = 0; t < kTileW; ++t) {
                if (t + 1 < kTileW) ld_init(t + 1, s4b[(t + 1) & 1]);
                const float4 (&s4)[8] = s4b[t & 1];
                const int k0 = (vw * kTileW + t) * 32;  // local column of the tile
                const int kk = k0 + lane;
                const uint32_t bi = vbase + kk < V ? binfo[tb * VA + vbase + kk] : 0u;
                const int bw = (int)(bi & 63u), roff = (int)(bi >> 6);
                const uint32_t bmask = (uint32_t)((((1ull << bw) - 1ull) << (roff & 3)) >> (32 * wq));
                // this view's final band in window wq -> its staging row (positions outside: 0)
                const float* se = sb + kk + (32 * wq - (roff & 3)) * RS;
#pragma unroll
                for (int q4 = 0; q4 < 8; ++q4) {
                    float rv[4];
#pragma unroll
                    for (int j = 0; j < 4; ++j) {
                        const int p = 4 * q4 + j;
                        rv[j] = (bmask & (1u << p)) ? se[p * RS] : 0.f;
                    }
                    *(float4*)(stg_w + lane * kStg + 4 * q4) = make_float4(rv[0], rv[1], rv[2], rv[3]);
                }
                __syncwarp();
#pragma unroll
                for (int m = 0; m < 8; ++m) {
                    const int i = 4 * m + sub;
                    const int oi = __shfl_sync(kFull, roff, i);
                    const uint32_t nib = __shfl_sync(kFull, bmask, i) >> (4 * ch);
                    const float4 f4 = *(const float4*)(stg_w + i * kStg + 4 * ch);
                    const float fv[4] = {f4.x, f4.y, f4.z, f4.w};
                    const float e0[4] = {s4[m].x, s4[m].y, s4[m].z, s4[m].w};
                    float d[4];
#pragma unroll
                    for (int j = 0; j < 4; ++j) d[j] = (nib & (1u << j)) ? fv[j] - e0[j] : 0.f;
                    if (vbase + k0 + i < V && (d[0] != 0.f || d[1] != 0.f || d[2] != 0.f || d[3] != 0.f))
                        red_add_v4(ez + (oi - (oi & 3)) + 32 * wq + 4 * ch, d[0], d[1], d[2], d[3]);
                }
                __syncwarp();
            }
            }
        } else if (is_delta) {
            // the image and the counters, then the next task's preparation (with the prior warp)
            for (int i = lane; i < tw * th && crank == 0; i += 32) {
                const int lx = i % tw, ly = i / tw;
                P.x[(size_t)(z + 1) * plane + (size_t)(gy0 + ly) * P.nx + gx0 + lx] = xt[cslot + ly * TW + lx];
            }
            if (lane == 0 && crank == 0) {
                P.sv_amount[(size_t)z * P.nsv + sv] = amount;
                atomicAdd(P.counters + 0, (unsigned long long)nactv);
                atomicAdd(P.counters + 1, (unsigned long long)(tw * th - nactv));
                atomicAdd(P.counters + 2, 1ull);
                atomicAdd(P.sum_delta, (double)amount);
            }
            finish_prepare(cb ^ 1);
        } else if (is_prior) {
            finish_prepare(cb ^ 1);
        }
        __syncthreads();
        if (PROF && threadIdx.x == 0 && crank == 0) {
            const long long tp4 = clock64();
            atomicAdd(P.tprof + 0, (unsigned long long)(tp1 - tp0));  // x tile, zero-skip, order
            atomicAdd(P.tprof + 1, (unsigned long long)(tp2 - tp1));  // SVB pack
            atomicAdd(P.tprof + 2, (unsigned long long)(tp3 - tp2));  // voxel loop
            atomicAdd(P.tprof + 3, (unsigned long long)(tp4 - tp3));  // write-back
            atomicAdd(P.tprof + 4, (unsigned long long)nactv);
            atomicAdd(P.tprof + 5, 1ull);
        }
    }
    if (MB && bt + 1 < nbatch) {  // grid barrier (bar.sync, fence + arrival, acquire spin, bar.sync)
        __syncthreads();
        if (threadIdx.x == 0) {
            __threadfence();
            atomicAdd(P.gbar, 1u);
            const unsigned target = (unsigned)(bt + 1) * gridDim.x;
            for (;;) {
                unsigned v;
                asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(P.gbar) : "memory");
                if (v >= target) break;
                __nanosleep(32);
            }
            __threadfence();
        }
        __syncthreads();
    }
    }
    if (CL == 2) cluster_sync_all();  // no CTA leaves while its peer may still write into it
}

// the dynamic shared-memory opt-in and carveout of a kernel, set once per (device, kernel) for
// the largest size seen (driver calls per launch would dominate short many-batch 2-D iterations)
cudaError_t ensure_smem_attr(const void* kern, int smem)
{
    static std::mutex mu;
    static std::map<std::pair<int, const void*>, int> done;
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) return e;
    std::lock_guard<std::mutex> lk(mu);
    int& have = done[{dev, kern}];
    if (have >= smem) return cudaSuccess;
    e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    if (e != cudaSuccess) return e;
    e = cudaFuncSetAttribute(kern, cudaFuncAttributePreferredSharedMemoryCarveout, 100);
    if (e != cudaSuccess) return e;
    have = smem;
    return cudaSuccess;
}

// A-record ring depth (voxels of cp.async lookahead): u8 records are 5 B/view, fp32 ones 17 B/view
// (>= 2: the loop holds the current voxel's stage and the next voxel's)
constexpr int ring_depth(bool u8) { return u8 ? 12 : 4; }

template <int VPT, bool U8, int NNB, int R, int CL, int KV>
auto pick_kernel(const IcdParams& p)
{
    // the phase profile (development aid) is built for the production variants only
    constexpr bool kProf = VPT == MBIR_WIDE_VPT && U8 && CL == 1;
    // several batches per launch: one CTA per task, exact single-voxel steps (api.cu launches the
    // other variants once per batch)
    constexpr bool kMB = CL == 1 && KV == 1;
    if (kMB && p.nbatch > 1)
        return p.theta2_pass ? k_svicd<VPT, U8, NNB, R, CL, KV, true, false, kMB>
                             : k_svicd<VPT, U8, NNB, R, CL, KV, false, false, kMB>;
    return p.theta2_pass ? k_svicd<VPT, U8, NNB, R, CL, KV, true, false, false>
           : (kProf && p.tprof) ? k_svicd<VPT, U8, NNB, R, CL, KV, false, kProf, false>
                                : k_svicd<VPT, U8, NNB, R, CL, KV, false, false, false>;
}

template <int VPT, bool U8, int NNB, int CL>
cudaError_t launch_t(const IcdParams& p, int gx, cudaStream_t st)
{
    constexpr int R = ring_depth(U8);
    // voxel pairs: uint8 A with one CTA per task (api.cu validates)
    constexpr bool kPairs = U8 && CL == 1;
    auto kern = (kPairs && p.kv == 2) ? pick_kernel<VPT, U8, NNB, R, CL, kPairs ? 2 : 1>(p)
                                      : pick_kernel<VPT, U8, NNB, R, CL, 1>(p);
    IcdParams q = p;
    q.lay = svicd_layout(p.rows, p.side, p.S2, NNB, p.A.VA, U8, R, p.nvw, VPT, p.V, CL);
    const int smem = q.lay.total;
    cudaError_t e = ensure_smem_attr((const void*)kern, smem);
    if (e != cudaSuccess) return e;
    const int threads = 32 * (p.nvw / CL + 2);
    if (CL == 1 && p.nbatch <= 1) {
        kern<<<gx, threads, smem, st>>>(q);
        return cudaGetLastError();
    }
    cudaLaunchConfig_t cfg{};
    cfg.gridDim = dim3(gx);
    cfg.blockDim = dim3(threads);
    cfg.dynamicSmemBytes = smem;
    cfg.stream = st;
    if (CL == 1) {  // several batches with grid barriers: every CTA must be resident
        cudaLaunchAttribute co[1];
        co[0].id = cudaLaunchAttributeCooperative;
        co[0].val.cooperative = 1;
        cfg.attrs = co;
        cfg.numAttrs = 1;
        return cudaLaunchKernelEx(&cfg, kern, q);
    }
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeClusterDimension;
    at[0].val.clusterDim.x = CL;
    at[0].val.clusterDim.y = 1;
    at[0].val.clusterDim.z = 1;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    return cudaLaunchKernelEx(&cfg, kern, q);
}

template <int VPT, bool U8, int NNB, int CL>
int resident_t(const IcdParams& p)
{
    auto kern = k_svicd<VPT, U8, NNB, ring_depth(U8), CL, 1, false, false, false>;
    const int smem = svicd_layout(p.rows, p.side, p.S2, NNB, p.A.VA, U8, ring_depth(U8), p.nvw, VPT, p.V, CL).total;
    if (cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, smem) != cudaSuccess) return -1;
    cudaFuncSetAttribute(kern, cudaFuncAttributePreferredSharedMemoryCarveout, 100);
    const int threads = 32 * (p.nvw / CL + 2);
    if (CL == 1) {
        int nb = 0, dev = 0, nsm = 0;
        if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, kern, threads, smem) != cudaSuccess) return -1;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
        return nb * nsm;
    }
    cudaLaunchConfig_t cfg{};
    cfg.gridDim = dim3(4 * 148);
    cfg.blockDim = dim3(threads);
    cfg.dynamicSmemBytes = smem;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeClusterDimension;
    at[0].val.clusterDim.x = CL;
    at[0].val.clusterDim.y = 1;
    at[0].val.clusterDim.z = 1;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    int ncl = 0;
    if (cudaOccupancyMaxActiveClusters(&ncl, kern, &cfg) != cudaSuccess) return -1;
    return ncl * CL;
}

// vpt: 1 (nviews <= 128) or MBIR_WIDE_VPT; cl: 1, or 2 (wide VPT only)
#define SVICD_DISPATCH1(FN, NNB_, U8_, ...)              \
    constexpr int W = MBIR_WIDE_VPT;                       \
    if (cl == 2) return FN<W, U8_, NNB_, 2>(__VA_ARGS__);  \
    if (vpt == 1) return FN<1, U8_, NNB_, 1>(__VA_ARGS__); \
    return FN<W, U8_, NNB_, 1>(__VA_ARGS__);

}  // namespace

#define SVICD_CAT2(a, b) a##_##b
#define SVICD_CAT(a, b) SVICD_CAT2(a, b)
#ifdef SVICD_NNB
// this translation unit's instantiations: one (neighbourhood, A type) pair (svicd_n*_*.cu; the
// kernel is split over four translation units so they compile in parallel)
int SVICD_CAT(svicd_resident, SVICD_SUFFIX)(const IcdParams& p, int vpt, int cl)
{
    SVICD_DISPATCH1(resident_t, SVICD_NNB, SVICD_U8, p)
}
cudaError_t SVICD_CAT(svicd_launch, SVICD_SUFFIX)(const IcdParams& p, int vpt, int cl, int grid, cudaStream_t st)
{
    SVICD_DISPATCH1(launch_t, SVICD_NNB, SVICD_U8, p, grid, st)
}
#endif

}  // namespace mbir
