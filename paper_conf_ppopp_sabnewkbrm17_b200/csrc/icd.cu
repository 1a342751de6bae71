// Fused SuperVoxel ICD update kernel for sm_100a, plus the
// theta2 precompute, forward projection and probe kernels that share its data layout.
//
// Paper: Alg. 1 is the per-voxel update; Alg. 3 runs it with
// intra-voxel, intra-SV and inter-SV parallelism over SV buffers
// created before and written back after the update.
//
// B200 design: one CTA per SM owns one (slice, SV) task at a time,
// persistent over the phase's task list.  Its view threads own VIEWS: view warp w, lane l owns
// views (w*VPT + t)*32 + l, t < VPT.  The SV buffer (e and w over the SV's sinogram band) lives
// in shared memory as [row = channel offset in band][view] with a view stride that is a multiple
// of 32, so a warp's 32 lanes always hit 32 distinct banks whatever the voxels' per-view offsets
// (conflict-free gather and scatter without atomics: a thread is the only writer of its views).
// Voxels of the SV are updated in a random order exactly as sequential ICD, two per step: the
// view warps gather both voxels' theta1 partials from the same e (their overlap H = sum w A_b A_a
// and w A were prepared in the previous step), warp-reduce and arrive on a named barrier; the
// prior warp derives delta_a, then theta1_b corrected by a's change and delta_b (q-GGMRF
// surrogate, reading R1), publishes them on a second barrier and computes the next pair's
// surrogate sums from a shared-memory x tile; the view warps scatter e -= A delta into their own
// views.  A records (uint8 codes + band offsets) are streamed R voxels ahead by per-thread
// cp.async.  theta2 = A^T W A is fixed by w and precomputed per (slice, voxel).  The SVB is
// packed from 16-byte-aligned band windows transposed through per-warp staging tiles, and written
// back as delta e = final - e_init with red.global.add.v4.f32, because same-colour SVs share
// sinogram entries.
#include "mbir_internal.h"

#include <cstdio>
#include <cstdlib>

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

// Neighbour slots of a prior-warp lane: half-warp h = lane >> 4 works on voxel a (h = 0) or b
// (h = 1) of a pair; its lane i owns neighbours i and i + 16 of the neighbourhood (reading R2):
// offset (dx, dy, dz), tile-index offset dt and weight w (0: no neighbour)
struct NbrLane {
    int dx[2], dy[2], dz[2], dt[2];
    float w[2];
};

// surrogate terms of a pair of consecutive voxels (a, b): a's sums, b's sums computed with a's
// OLD value, and -- if a is b's neighbour -- that neighbour's term (btab) and weight (bab)
struct PriPair {
    float sa, sxa, va, sb, sxb, vb, btab, bab;
};

// sum of NS (8 or 16) consecutive floats (16-byte aligned) with paired-fp32 adds, in a fixed
// order (every warp of the task gets the same bits)
template <int NS>
__device__ __forceinline__ float sum_slots(const float* r)
{
    const float4 a = ((const float4*)r)[0], b = ((const float4*)r)[1];
    float2 s = __fadd2_rn(__fadd2_rn(make_float2(a.x, a.y), make_float2(a.z, a.w)),
                          __fadd2_rn(make_float2(b.x, b.y), make_float2(b.z, b.w)));
    if (NS == 16) {
        const float4 c = ((const float4*)r)[2], d = ((const float4*)r)[3];
        s = __fadd2_rn(s, __fadd2_rn(__fadd2_rn(make_float2(c.x, c.y), make_float2(c.z, c.w)),
                                     __fadd2_rn(make_float2(d.x, d.y), make_float2(d.z, d.w))));
    }
    return s.x + s.y;
}

template <bool B>
struct BoolTag {
    static constexpr bool value = B;
};

// dequantised codes i, i + 1 of a packed word as a channel pair: 2 PRMT + 1 FADD2
__device__ __forceinline__ float2 dq2(uint32_t word, int i)
{
    const float2 m = make_float2(__uint_as_float(__byte_perm(word, 0x4B000000u, 0x7440u | (uint32_t)i)),
                                 __uint_as_float(__byte_perm(word, 0x4B000000u, 0x7441u + (uint32_t)i)));
    return __fadd2_rn(m, make_float2(-8388608.f, -8388608.f));
}

// A values of a voxel re-indexed to another voxel's channels: r[i] = A[i + d] (0 outside), as
// channel pairs
template <bool U8>
__device__ __forceinline__ void shifted(uint32_t cw, const float2 (&a)[2], int d, float2 (&r)[2])
{
    if (U8) {
        // one PRMT: byte i of s = byte i + d of cw, or 0 (selector nibble 4 = byte 0 of the zero
        // operand); the selector nibbles are read out of 0x444432104444 at nibble 4 + d
        const int dc = max(-4, min(4, d));
        const uint32_t sel = (uint32_t)(0x444432104444ull >> (16 + 4 * dc));
        const uint32_t s = __byte_perm(cw, 0u, sel);
        r[0] = dq2(s, 0);
        r[1] = dq2(s, 2);
        return;
    }
    const float v[4] = {a[0].x, a[0].y, a[1].x, a[1].y};
    float q[4];
#pragma unroll
    for (int i = 0; i < 4; ++i) {
        const int j = i + d;
        q[i] = j == 0 ? v[0] : j == 1 ? v[1] : j == 2 ? v[2] : j == 3 ? v[3] : 0.f;
    }
    r[0] = make_float2(q[0], q[1]);
    r[1] = make_float2(q[2], q[3]);
}

// this thread's VPT adjacent records (apos) from a stage as raw words (CW = 1: a uint8 code word
// per view; CW = 4: fp32 values), and the band offsets packed in one word (VPT bytes)
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
    if (VPT == 2) ob = ((const uint16_t*)(stg + off_in_stage))[tp];
    if (VPT == 1) ob = stg[off_in_stage + tp];
}

// prior warp: PriPair for voxels (i0, i0+1) of the visiting order from the current x tile.
// Alg1:7's q-GGMRF surrogate sums sb = sum_r b_r phi(v - x_r), sx = sum_r b_r phi(v - x_r) x_r
// over the neighbourhood (free boundary: off-image neighbours contribute nothing), voxel a on
// lanes 0-15 and voxel b (with a's OLD value) on lanes 16-31, two neighbours per lane, so both
// voxels' terms are one latency chain and a 4-level half-warp reduction.
__device__ __forceinline__ void prior_pair(const int* tof, int i0, int nact, const float* xt, int cslot,
                                           int TW, int gx0, int gy0, int zg, const IcdParams& P,
                                           const NbrLane& nb, int lane, PriPair* out)
{
    const bool hasb = i0 + 1 < nact;
    const int ta = tof[i0], tb = hasb ? tof[i0 + 1] : ta;
    const int tv = lane < 16 ? ta : tb;
    const int lx = tv & 255, ly = tv >> 8;
    const int c0 = cslot + ly * TW + lx;
    const float v = xt[c0];
    float sb = 0.f, sx = 0.f, btn = 0.f, bwn = 0.f;  // btn, bwn: this lane's term / weight whose
    bool mine = false;                               // neighbour is voxel a
    const int dxa = (ta & 255) - lx, dya = (ta >> 8) - ly;  // a relative to this half's voxel
#pragma unroll
    for (int k = 0; k < 2; ++k) {
        const int gx = gx0 + lx + nb.dx[k], gy = gy0 + ly + nb.dy[k], gz = zg + nb.dz[k];
        if (nb.w[k] != 0.f && gx >= 0 && gx < P.nx && gy >= 0 && gy < P.ny && gz >= 0 && gz < P.nz_total) {
            const float xr = xt[c0 + nb.dt[k]];
            const float bt = nb.w[k] * phi_f(P.pc, v - xr);
            sb += bt;
            sx += bt * xr;
            if (nb.dz[k] == 0 && nb.dx[k] == dxa && nb.dy[k] == dya) {
                btn = bt;
                bwn = nb.w[k];
                mine = true;
            }
        }
    }
#pragma unroll
    for (int o = 8; o > 0; o >>= 1) {
        sb += __shfl_xor_sync(kFull, sb, o);
        sx += __shfl_xor_sync(kFull, sx, o);
    }
    // a's neighbour term in b's sums (a and b are distinct voxels, so only lanes >= 16 can own it)
    const unsigned who = __ballot_sync(kFull, mine && lane >= 16 && hasb);
    const int src = who ? __ffs(who) - 1 : 0;
    const float btab = __shfl_sync(kFull, btn, src);
    const float bab = __shfl_sync(kFull, bwn, src);
    const float sbb = __shfl_sync(kFull, sb, 16), sxb = __shfl_sync(kFull, sx, 16), vb = __shfl_sync(kFull, v, 16);
    if (lane == 0) {
        PriPair pp{sb, sx, v, 0.f, 0.f, 0.f, 0.f, 0.f};
        if (hasb) {
            pp.sb = sbb;
            pp.sxb = sxb;
            pp.vb = vb;
            if (who) {
                pp.btab = btab;
                pp.bab = bab;
            }
        }
        *out = pp;
    }
}

// ---- mbarrier, cp.async and L2-prefetch helpers ----
__device__ __forceinline__ uint32_t smem_u32(const void* p)
{
    return (uint32_t)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count)
{
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t* bar)
{
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
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
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_async_wait()
{
    asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory");
}

// ---- thread-block-cluster helpers (CL = 2: the two CTAs of a cluster split an SV's views) ----
__device__ __forceinline__ uint32_t cluster_rank()
{
    uint32_t r;
    asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
    return r;
}
// shared::cluster address of the same smem location in CTA `rank` of the cluster
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
// arrive on an mbarrier of the peer CTA; release at cluster scope orders this thread's earlier
// st.shared::cluster writes before the arrival
__device__ __forceinline__ void mbar_arrive_peer(uint32_t a)
{
    asm volatile("mbarrier.arrive.release.cluster.shared::cluster.b64 _, [%0];" ::"r"(a) : "memory");
}
// wait for a phase with acquire at cluster scope (sees the peer's released writes)
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

__host__ __device__ inline int align16(int b) { return (b + 15) & ~15; }

// row stride (floats) of a view warp's 32-row transpose staging tile: 16-byte rows, so a lane moves
// 4 window positions with one STS.128 / LDS.128; every quarter-warp (one shared-memory wavefront
// of a 128-bit access) then touches 8 distinct 4-bank groups, on the put (lanes span rows and
// float4 chunks) and on the read (lane k reads its own row)
constexpr int kStg = 36;

// the update kernel's SVB column stride: the most views one CTA can hold (VPT = 1: 6 view warps
// of 32; VPT >= 2: 768 views = 24 / VPT view warps, / CL), fixed at compile time whatever the
// actual view count
__host__ __device__ constexpr int svb_stride(int vpt, int cl = 1) { return (vpt == 1 ? 192 : 768) / cl; }

// partial-sum slots per quantity in the pair exchange (>= view warps of a task)
__host__ __device__ constexpr int red_slots(int vpt) { return vpt == 2 ? 16 : 8; }

// pair-exchange buffers of the update kernel (red partials / prior terms): the cluster variant
// needs 3 (a CTA can run one pair ahead of its peer), 4 keeps the index a mask
constexpr int kPairBufs = 4;

// A-record stage: U8: codes u32[VL] then offsets u8[VL]; fp32: float4[VL] then offsets u8[VL];
// VL = VA / cl record positions (this CTA's views)
__host__ __device__ inline SmemLayout smem_layout(int rows, int Vs, int side, int S2, int nnb,
                                                  int VA, bool u8, int nstage, int nvw, int cl)
{
    SmemLayout L;
    const int TW = side + 2;
    const int nzt = nnb == 26 ? 3 : 1;
    const int VL = VA / cl, nvl = nvw / cl;
    int o = 0;
    L.sb_e = o;  o = align16(o + rows * Vs * 4);
    L.sb_w = o;  o = align16(o + rows * Vs * 4);
    L.xt = o;    o = align16(o + nzt * TW * TW * 4);
    L.list = o;  o = align16(o + S2 * 4);
    L.flags = o; o = align16(o + S2 * 4);
    L.tof = o;   o = align16(o + S2 * 4);
    L.red = o;   o = align16(o + kPairBufs * 3 * 16 * 4);  // [bufs][3 quantities][<= 16 view warps]
    L.pri = o;   o = align16(o + kPairBufs * (int)sizeof(PriPair));
    L.vscale = o; o = align16(o + S2 * 4);
    L.vth2 = o;  o = align16(o + S2 * 4);
    L.misc = o;  o = align16(o + 16 * 4);
    L.off_in_stage = VL * (u8 ? 4 : 16);
    L.stage_bytes = align16(L.off_in_stage + VL);
    // the A-record ring (voxel loop) and the transpose staging tiles (pack, write-back) are never
    // live at the same time: they share one region
    L.astage = o;
    L.staging = o;
    o = align16(o + max(nstage * L.stage_bytes, nvl * 32 * kStg * 4));  // staging: a 32 x kStg tile per view warp
    // pair[kPairBufs], task[1]
    L.mbar = o;  o = align16(o + (kPairBufs + 1) * 8);
    L.binfo = o; o = align16(o + 2 * VL * 4);           // band (row offset << 5 | width), 2 tasks
    L.total = o;
    return L;
}

// band of task tk for this CTA's views vbase + k, k = k0, k0 + stride, ... < VL (and < V) into
// dst[k] = ((vbase + k)*M + start) << 5 | width
__device__ __forceinline__ void band_info(const IcdParams& P, int tk, uint32_t* dst, int vbase, int VL,
                                          int k0, int stride)
{
    const int sv = tk & 16383;
    for (int k = k0; k < VL && vbase + k < P.V; k += stride) {
        const int kg = vbase + k;
        const int r = kg * P.M + P.A.band_start[(size_t)sv * P.V + kg];
        const int wd = P.A.band_width[(size_t)sv * P.V + kg];
        dst[k] = ((uint32_t)r << 5) | (uint32_t)wd;
    }
}

// CL = 1: one CTA per SM owns a whole (slice, SV) task.  CL = 2: a 2-CTA cluster owns the task,
// each CTA holding half the views (its half of the SVB and of every A record), two clusters'
// CTAs per SM; per voxel pair the CTAs exchange their partial sums through distributed shared
// memory, so both derive the same deltas.  Two independent tasks per SM let one CTA's pack and
// write-back overlap the other's voxel loop.
// CL = 1: one CTA per SM of <= 6 (VPT 1, 4) or 12 (VPT 2) view warps + the prior warp; CL = 2:
// two CTAs of 3 view warps + the prior warp per SM (8 warps: the full register budget)
template <int VPT, bool U8, int NNB, int R, int CL, bool PROF>
__global__ void __launch_bounds__(CL == 2 ? (VPT == 2 ? 224 : 128) : (VPT == 2 ? 416 : 224), CL == 1 ? 1 : 2) k_icd_sv(const IcdParams P)
{
    extern __shared__ __align__(16) unsigned char smem[];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const int nvw = P.nvw;              // view warps of the whole task (both CTAs)
    const int nvl = nvw / CL;           // view warps of this CTA
    const uint32_t crank = CL == 1 ? 0u : cluster_rank();
    // warp roles: nvl view warps and the prior warp, which also produces the A-record stream
    // (TMA) and the next task's band info.  Warps w and w + 4 share a scheduler (SMSP); with >= 3
    // view warps the prior warp is warp 3, so the view warps spread evenly over SMSPs 0-2 (and 3
    // when nvl is small).
    const int prior_w = nvl >= 3 ? 3 : nvl;
    const bool is_prior = warp == prior_w, is_view = !is_prior;
    const int vw = is_view ? (warp < prior_w ? warp : warp - 1) : 0;  // local view-warp index
    const int gvw = (int)crank * nvl + vw;                             // view-warp index in the task
    const int V = P.V, M = P.M, S2 = P.S2, side = P.side;
    const int VL = P.A.VA / CL;          // record positions / SVB columns of this CTA
    const int vbase = (int)crank * VL;   // first view (and record position) of this CTA
    constexpr int VS = svb_stride(VPT, CL);  // SVB view stride: compile-time, so row offsets are immediates
    constexpr int NSL = red_slots(VPT);      // pair-exchange slots per quantity
    const SmemLayout& L = P.lay;
    float* sb_e = (float*)(smem + L.sb_e);
    float* sb_w = (float*)(smem + L.sb_w);
    float* xt = (float*)(smem + L.xt);
    int* list = (int*)(smem + L.list);
    int* flags = (int*)(smem + L.flags);
    int* tof = (int*)(smem + L.tof);  // visiting order as packed (ly << 8 | lx)
    float* red = (float*)(smem + L.red);
    PriPair* pri = (PriPair*)(smem + L.pri);
    float* vscale = (float*)(smem + L.vscale);
    float* vth2 = (float*)(smem + L.vth2);
    uint64_t* mbar = (uint64_t*)(smem + L.mbar);
    unsigned char* astage = smem + L.astage;
    float* stg_w = (float*)(smem + L.staging) + vw * 32 * kStg;
    const int TW = side + 2;
    const int zc = (NNB == 26) ? 1 : 0;  // centre slice of the x tile
    const size_t plane = (size_t)P.nx * P.ny;
    uint64_t* pairbar = mbar;              // [kPairBufs] (CL = 2): both CTAs' partials + prior terms
    uint64_t* taskbar = pairbar + kPairBufs;  // (CL = 2, rank 1): the next task id has arrived

    for (int i = threadIdx.x; i < kPairBufs * 3 * NSL; i += blockDim.x) red[i] = 0.f;  // slots >= nvw stay zero
    // SVB rows outside a visit's band are never packed: start them finite (zero)
    for (int i = threadIdx.x; i < (L.sb_w - L.sb_e) / 16; i += blockDim.x) {
        ((float4*)(smem + L.sb_e))[i] = make_float4(0.f, 0.f, 0.f, 0.f);
        ((float4*)(smem + L.sb_w))[i] = make_float4(0.f, 0.f, 0.f, 0.f);
    }
    if (threadIdx.x == 0) {
        for (int b = 0; b < kPairBufs; ++b) mbar_init(pairbar + b, nvw);  // all view warps of the task
        mbar_init(taskbar, 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    // per-thread view ownership: (task) view-warp g, lane l owns views (g*VPT + t)*32 + l, held in
    // SVB column (vw*VPT + t)*32 + l of its CTA
    int kv[VPT];
    bool kval[VPT];
#pragma unroll
    for (int t = 0; t < VPT; ++t) {
        kv[t] = (vw * VPT + t) * 32 + lane;
        kval[t] = is_view && vbase + kv[t] < V;
    }
    uint32_t gseq = 0;  // running voxel sequence number of this CTA: A stage = gseq % R
    uint32_t pseq = 0;  // running voxel-pair number: exchange buffer pseq % kPairBufs
    uint32_t ntask = 0; // tasks with a voxel loop so far (task-id handoff parity, CL = 2)
    // prior-warp lane r owns neighbour r: its offset and weight live in registers (a per-lane
    // __constant__ index would serialise in the constant cache on every voxel)
    NbrLane nb;
#pragma unroll
    for (int k = 0; k < 2; ++k) {
        const int r = (lane & 15) + 16 * k;
        const bool ok = r < P.pc.nnb;
        nb.dx[k] = ok ? P.pc.dx[r] : 0;
        nb.dy[k] = ok ? P.pc.dy[r] : 0;
        nb.dz[k] = ok ? P.pc.dz[r] : 0;
        nb.w[k] = ok ? P.pc.b[r] : 0.f;
        nb.dt[k] = (nb.dz[k] * (side + 2) + nb.dy[k]) * (side + 2) + nb.dx[k];
    }

    // this launch's batch: flat tasks [start, end) of the phase list (sched.cu k_flatten),
    // pulled one at a time by the persistent CTAs (dynamic distribution, Alg3:4 / T3)
    const int tstart = P.brange[0], tend = P.brange[1];
    // s_task[0]: first task; s_task[1 + (n & 1)]: the task after task n (fetched one ahead by
    // rank 0 and, CL = 2, stored into both CTAs; alternating slots so a write for task n + 1
    // never meets a read of task n's)
    int* s_task = (int*)(smem + L.misc);
    uint32_t* binfo = (uint32_t*)(smem + L.binfo);  // [2][VL]: this task's / the next task's band
    // publish a task index (rank 0 only) into slot i of both CTAs
    auto publish_task = [&](int i, int v) {
        s_task[i] = v;
        if (CL == 2) st_peer_u32(peer_addr(s_task + i, 1), (uint32_t)v);
    };
    if (CL == 2) cluster_sync_all();  // peer smem (mbarriers, red) initialised before any remote access
    // the next task of the launch's list; with the zero-skip pre-filter (P.keep), tasks whose
    // whole tile is zero are accounted as skipped visits here and never reach a CTA's pipeline
    auto fetch_task = [&]() {
        int q = tstart + atomicAdd(P.fetch, 1);
        while (P.keep && q < tend && !P.keep[q]) {
            const int tkq = P.flat[q];
            const int zq = tkq >> 14, svq = tkq & 16383;
            const int twq = min(side, P.nx - (svq % P.nsvx) * side), thq = min(side, P.ny - (svq / P.nsvx) * side);
            P.sv_amount[(size_t)zq * P.nsv + svq] = 0.f;
            atomicAdd(P.counters + 1, (unsigned long long)(twq * thq));
            atomicAdd(P.counters + 2, 1ull);
            atomicAdd(P.counters + 3, 1ull);
            q = tstart + atomicAdd(P.fetch, 1);
        }
        return q;
    };
    if (threadIdx.x == 0 && crank == 0) publish_task(0, fetch_task());
    if (CL == 2) cluster_sync_all(); else __syncthreads();
    int q = s_task[0];
    if (q < tend) band_info(P, P.flat[q], binfo, vbase, VL, threadIdx.x, blockDim.x);
    int tb = 0;  // binfo buffer of the current task
    int nslot = 1;  // s_task slot of the next task
    for (;; q = s_task[nslot], nslot ^= 3, tb ^= 1) {
        if (q >= tend) break;
        const int tk = P.flat[q];
        const int z = tk >> 14, sv = tk & 16383;  // local slice, SV
        // development aid (env MBIR_TRACE, profiled build only): clock64 stamps of every voxel pair
        // of one SV visit (CTA 0's sixth task of the first launch), slot 1 + 16 * pair + k
        const bool TR = PROF && P.trace && blockIdx.x == 0 && ntask == 5 && *(volatile unsigned long long*)P.trace == 0ull;
        auto stamp = [&](int pair, int k) {
            if (TR) P.trace[1 + 16 * pair + k] = (unsigned long long)clock64();
        };
        if (threadIdx.x == 0) stamp(60, 0);
        const int zg = P.z_offset + z;            // global slice
        const int bx = sv % P.nsvx, by = sv / P.nsvx;
        const int gx0 = bx * side, gy0 = by * side;
        const int tw = min(side, P.nx - gx0), th = min(side, P.ny - gy0);

        long long tp0 = 0, tp1 = 0, tp1b = 0, tp2 = 0, tp3 = 0;
        if (PROF && P.tprof && threadIdx.x == 0) tp0 = clock64();
        // ---- 1. x tile (+1 halo ring, +-1 slice in 3-D) into shared memory
        {
            // all of a thread's loads first (clamped, always in bounds), then the zeroing of
            // off-image entries and the stores: the loads are in flight together
            constexpr int XMAX = 4;  // tile entries per thread and round
            const int ntile = (NNB == 26 ? 3 : 1) * TW * TW;
            for (int i0 = 0; i0 < ntile; i0 += XMAX * blockDim.x) {
            float xv[XMAX];
            bool inb[XMAX];
#pragma unroll
            for (int u = 0; u < XMAX; ++u) {
                const int i = i0 + threadIdx.x + u * blockDim.x;
                const int tz = i / (TW * TW), r = i % (TW * TW), ty = r / TW, tx = r % TW;
                const int gx = gx0 - 1 + tx, gy = gy0 - 1 + ty;
                const int zs = (NNB == 26) ? z + tz : z + 1;  // storage slice (halo at 0, nz+1)
                inb[u] = i < ntile && gx >= 0 && gx < P.nx && gy >= 0 && gy < P.ny;
                const int cx = min(max(gx, 0), P.nx - 1), cy = min(max(gy, 0), P.ny - 1);
                xv[u] = i < ntile ? P.x[(size_t)min(zs, P.nz_local + 1) * plane + (size_t)cy * P.nx + cx] : 0.f;
            }
#pragma unroll
            for (int u = 0; u < XMAX; ++u) {
                const int i = i0 + threadIdx.x + u * blockDim.x;
                if (i < ntile) xt[i] = inb[u] ? xv[u] : 0.f;
            }
            }
        }
        __syncthreads();

        // ---- 2. zero-skip predicate at visit start (reading R9): slot v kept iff valid
        //         and (skip inactive or x_j or a neighbour is non-zero)
        int keep = 0;
        const int v0 = threadIdx.x;
        if (v0 < S2) {
            const int lx = v0 % side, ly = v0 / side;
            if (lx < tw && ly < th) {
                keep = 1;
                if (P.zero_skip_active) {
                    keep = xt[(zc * TW + ly + 1) * TW + lx + 1] != 0.f;
                    for (int r = 0; r < P.pc.nnb && !keep; ++r) {
                        const int gx = gx0 + lx + P.pc.dx[r], gy = gy0 + ly + P.pc.dy[r];
                        const int gz = zg + P.pc.dz[r];
                        if (gx < 0 || gx >= P.nx || gy < 0 || gy >= P.ny || gz < 0 || gz >= P.nz_total) continue;
                        keep = xt[((zc + P.pc.dz[r]) * TW + ly + 1 + P.pc.dy[r]) * TW + lx + 1 + P.pc.dx[r]] != 0.f;
                    }
                }
            }
            flags[v0] = keep;
        }
        const int nact = __syncthreads_count(keep);
        if (nact == 0) {  // the whole SV is zero-skipped: account for it and take the next task
            if (threadIdx.x == 0 && crank == 0) {
                P.sv_amount[(size_t)z * P.nsv + sv] = 0.f;
                atomicAdd(P.counters + 1, (unsigned long long)(tw * th));
                atomicAdd(P.counters + 2, 1ull);
                atomicAdd(P.counters + 3, 1ull);
                publish_task(nslot, fetch_task());
            }
            if (CL == 2) cluster_sync_all(); else __syncthreads();
            if (s_task[nslot] < tend)
                band_info(P, P.flat[s_task[nslot]], binfo + (tb ^ 1) * VL, vbase, VL, threadIdx.x, blockDim.x);
            continue;  // the next task's x-tile barrier orders these writes before its pack
        }

        // ---- 3. visiting order: random permutation of the tile, compacted to the kept
        //         voxels with a warp ballot; per-voxel scale and theta2 staged in smem; the
        //         prior warp's lane 0 then starts the TMA ring of A records (R voxels ahead)
        const size_t arec = (size_t)sv * S2;  // first A record of this SV
        // view thread tp: asynchronous copy of its own slice of voxel j's record (this CTA's part)
        // into stage (gseq + j) % R, one commit group per voxel (empty past the visit's end).  A
        // thread reads back only what it copied (VPT = 1: its lane quad's offset word), so the
        // A stream needs no cross-warp synchronisation: per-thread LDGSTS + wait_group.
        // (per-task bases: this thread's slice of the SV's records in global memory and of a stage)
        constexpr int CB = U8 ? 4 : 16;  // record bytes per view position
        const int tpm = vw * 32 + lane;
        const unsigned char* g_code = (const unsigned char*)(U8 ? (const void*)P.A.codes : (const void*)P.A.vals) +
                                      ((size_t)arec * P.A.VA + vbase + tpm * VPT) * CB;
        const unsigned char* g_off = P.A.off + (size_t)arec * P.A.VA + vbase + tpm * VPT;
        // record of voxel j (slot v = list[j]) into ring stage `stg`
        auto copy_record_to = [&](int j, int stg, int v) {
            if (j < nact) {
                unsigned char* st = astage + stg * L.stage_bytes;
                const unsigned char* gc = g_code + (size_t)v * (P.A.VA * CB);
                if (U8) {
                    if (VPT == 4)
                        cp_async16(st + tpm * 16, gc);
                    else if (VPT == 2)
                        cp_async8(st + tpm * 8, gc);
                    else
                        cp_async4(st + tpm * 4, gc);
                } else {
#pragma unroll
                    for (int t = 0; t < VPT; ++t) cp_async16(st + (tpm * VPT + t) * 16, gc + t * 16);
                }
                // offsets: VPT bytes per thread, copied as 4-byte words by every (4 / VPT)-th lane
                if ((tpm & (4 / VPT - 1)) == 0)
                    cp_async4(st + L.off_in_stage + tpm * VPT, g_off + (size_t)v * P.A.VA);
            }
            cp_async_commit();
        };
        const int sbase = (int)(gseq % (uint32_t)R);  // ring stage of this visit's voxel 0
        auto copy_record = [&](int j, int tp) {
            (void)tp;
            copy_record_to(j, (sbase + j) % R, j < nact ? list[j] : 0);
        };
        if (is_prior) {
            // one of NPERM host-drawn random permutations of the tile, chosen per
            // (seed, iteration, slice, SV) visit; identity (raster order) in deterministic mode
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
                    list[p] = v;
                    tof[p] = ((v / side) << 8) | (v % side);  // packed (ly, lx): no div in the loop
                }
                n += __popc(m);
            }
            __syncwarp();
            for (int i = lane; i < nact; i += 32) {
                const int v = list[i];
                vscale[i] = P.A.scale[arec + v];
                vth2[i] = P.theta2[((size_t)z * P.nsv + sv) * S2 + v];
            }
            __syncwarp();
            if (lane == 0) {
                // the next task (rank 0 fetches it; CL = 2 hands it to rank 1 through DSMEM + an
                // mbarrier arrival)
                if (crank == 0) {
                    publish_task(nslot, fetch_task());
                    if (CL == 2) mbar_arrive_peer(peer_addr(taskbar, 1));
                }
            }
        }

        if (PROF && P.tprof && threadIdx.x == 0) tp1 = clock64();
        if (threadIdx.x == 0) stamp(60, 1);
        // ---- 4. view threads: SVB pack (coalesced 128-byte band rows, transposed by shuffles);
        //         e_init rows go to this CTA's L2-resident scratch tile for the write-back
        float* scr = P.scratch + (size_t)blockIdx.x * (size_t)P.Vs * 32;
        if (is_view) {
            const float* wz = P.w + (size_t)z * V * M;
            float* ez = P.e + (size_t)z * V * M;
            // Each band row is read as the 16-byte-aligned 32-float window that contains it (the
            // slice base is 16-byte aligned, V*M % 4 == 0): 8 lanes x float4 per row, 4 rows per
            // LDG.128, so a 32-view tile of w and e is 16 vector loads (few requests in flight).
            // The windows go through the warp's staging tile with a row stride of 33 floats: the
            // put (lanes span window position p = 4ch + j and row i = 4m + sub) and the read (lane
            // k walks its own row's positions) both touch 32 distinct banks, and band column
            // c = p - s_k goes to sb[c][k] (bank k).  Only band columns are written: the rows past
            // a view's band keep finite stale values that only ever meet zero A entries.
            // e_init windows go to this CTA's L2-resident scratch tile for the write-back.
            // Two tiles are in flight: tile t + 1's loads are issued before tile t is staged.
            const int sub = lane >> 3, ch = lane & 7;  // row-in-quad and float4 chunk of this lane
            auto issue = [&](int t, bool isw, float4 (&v4)[8]) {
                const int k0 = (vw * VPT + t) * 32;  // local column of the tile's first view
                const int kk = k0 + lane;
                const uint32_t bi = vbase + kk < V ? binfo[tb * VL + kk] : 0u;
                const int bwt = (int)(bi & 31u), rot = (int)(bi >> 5);
#pragma unroll
                for (int m = 0; m < 8; ++m) {
                    const int i = 4 * m + sub;
                    const int oi = __shfl_sync(kFull, rot, i);
                    // unconditional loads (no consumer until the staging, so all 8 are in flight):
                    // the whole aligned window is read even past the band (padded views read the
                    // slice start); only band positions are ever stored, and the sinogram
                    // allocations carry 32 floats of tail padding for the last row's window
                    const int s = oi & 3;
                    const size_t a4 = (size_t)(oi - s) + 4 * ch;
                    if (isw)
                        v4[m] = __ldg((const float4*)(wz + a4));
                    else
                        v4[m] = __ldcg((const float4*)(ez + a4));
                }
            };
            auto finish = [&](int t, bool isw, const float4 (&v4)[8]) {
                const int k0 = (vw * VPT + t) * 32;
                const int kk = k0 + lane;
                const uint32_t bi = vbase + kk < V ? binfo[tb * VL + kk] : 0u;
                const int bwt = (int)(bi & 31u), sk = (int)(bi >> 5) & 3;
                const uint32_t bmask = ((1u << bwt) - 1u) << sk;  // band's window positions
                if (!isw) {
#pragma unroll
                    for (int m = 0; m < 8; ++m) __stcg((float4*)(scr + (k0 + 4 * m + sub) * 32 + 4 * ch), v4[m]);
                }
                float* d = (isw ? sb_w : sb_e) + kk - sk * VS;  // + p * VS = band column p - sk of view kk
#pragma unroll
                for (int m = 0; m < 8; ++m) *(float4*)(stg_w + (4 * m + sub) * kStg + 4 * ch) = v4[m];
                __syncwarp();
#pragma unroll
                for (int q4 = 0; q4 < 8; ++q4) {
                    const float4 r = *(const float4*)(stg_w + lane * kStg + 4 * q4);
                    const float rv[4] = {r.x, r.y, r.z, r.w};
#pragma unroll
                    for (int j = 0; j < 4; ++j)
                        if (bmask & (1u << (4 * q4 + j))) d[(4 * q4 + j) * VS] = rv[j];
                }
                __syncwarp();
            };
            // software pipeline over the VPT tiles: tile t + 1's 16 window loads are in flight
            // while tile t is staged
            float4 wa[2][8], ea[2][8];
            issue(0, true, wa[0]);
            issue(0, false, ea[0]);
#pragma unroll
            for (int t = 0; t < VPT; ++t) {
                if (t + 1 < VPT) {
                    issue(t + 1, true, wa[(t + 1) & 1]);
                    issue(t + 1, false, ea[(t + 1) & 1]);
                }
                finish(t, true, wa[t & 1]);
                finish(t, false, ea[t & 1]);
            }
            if (PROF && P.tprof && threadIdx.x == 0) tp1b = clock64();
        }
        __syncthreads();

        if (PROF && P.tprof && threadIdx.x == 0) tp2 = clock64();
        if (threadIdx.x == 0) stamp(60, 2);
        // ---- 5. sequential-exact voxel loop, TWO voxels (a, b) per barrier.  Both are gathered
        //         from the same state of e, together with the overlap H = sum w A_b A_a over their
        //         shared sinogram entries; after the barrier every warp computes delta_a, then
        //         theta1_b corrected for a's update (theta1_b' = theta1_b + s_b s_a delta_a H, the
        //         exact change of e between them), the prior of b corrected if a is b's
        //         neighbour, then delta_b -- exactly sequential ICD in the visiting order.
        float amount = 0.f;
        const int cslot = (zc * TW + 1) * TW + 1;  // tile index of local (0,0)
        // Two named barriers per pair: A (1) -- the view warps' partial sums of the pair are in
        // `red` (view warps arrive, the prior warp waits); B (2) -- the prior warp has published the
        // pair's two deltas (prior warp arrives, view warps wait).  Only the prior warp evaluates
        // the delta chain; the view warps prepare the next pair's e-independent state (records, w,
        // w*A, the overlap H) while it runs, then scatter, then gather the next pair's e.
        const int npair_threads = (nvl + 1) * 32;  // view warps + prior warp
        float* dslot = (float*)(smem + L.misc) + 4;  // [2 pairs][2]: scale_a*delta_a, scale_b*delta_b
        if (is_view) {
            const int tp = vw * 32 + lane;  // this thread's record position in a stage
            // Per-pair state of a view thread, for its VPT views: band offsets of a and b (packed
            // bytes), their A records (uint8 code words, or fp32 values as bits), w*A_a, w*A_b on
            // their own channels (channel pairs (0,1), (2,3) for the paired-fp32 FFMA2/FMUL2 of
            // sm_100), and the warp-reduced overlap H = sum w A_b A_a.  None of it depends on e.
            constexpr int CW = U8 ? 1 : 4;  // record words per view
            struct PairState {
                uint32_t oa, ob;
                uint32_t ca[VPT][CW], cb[VPT][CW];
                float2 wa[VPT][2], wb[VPT][2];
                float hh;
                int sj;      // ring stage of voxel j (the pair's first voxel)
                int lv[2];   // list[j + R], list[j + 1 + R]: the records copied into its stages
            };
            // A values of a record as channel pairs
            auto avals = [&](const uint32_t (&c)[CW], float2 (&f)[2]) {
                if (U8) {
                    f[0] = dq2(c[0], 0);
                    f[1] = dq2(c[0], 2);
                } else {
                    f[0] = make_float2(__uint_as_float(c[0]), __uint_as_float(c[CW > 1 ? 1 : 0]));
                    f[1] = make_float2(__uint_as_float(c[CW > 2 ? 2 : 0]), __uint_as_float(c[CW > 3 ? 3 : 0]));
                }
            };
            auto off_of = [&](uint32_t packed, int t) { return (int)((packed >> (8 * t)) & 255u); };
            // voxels j, j + 1 of the visiting order -> ps.  A pair without a second voxel (the
            // last step of an odd visit, hb = false) gets a dummy b with zero A on a's channels:
            // its theta1 and H vanish, its delta is 0, and its scatter rewrites a's entries with
            // the same values -- no branches on the pair's shape.
            auto prep = [&](int j, bool hb, PairState& ps) {
                const long long tf0 = (PROF && P.tprof) ? clock64() : 0;
                // this thread's copies of voxels j, j + 1 have landed (R voxels' groups are in
                // flight: j .. j + R - 1)
                cp_async_wait<R - 2>();
                if (VPT != 4) __syncwarp();  // offset words copied by another lane of the warp
                if (PROF && P.tprof && lane == 0)   // development aid: A-stream wait
                    atomicAdd(P.tprof + 22 + (j >= R), (unsigned long long)(clock64() - tf0));
                const int sb1 = ps.sj + 1 == R ? 0 : ps.sj + 1;
                const unsigned char* sta = astage + ps.sj * L.stage_bytes;
                const unsigned char* stb = astage + sb1 * L.stage_bytes;
                // the slots of the records that will refill these stages (read early: the copy
                // after the scatter then needs no shared-memory round trip)
                ps.lv[0] = j + R < nact ? list[j + R] : 0;
                ps.lv[1] = j + 1 + R < nact ? list[j + 1 + R] : 0;
                load_words<VPT, CW>(sta, L.off_in_stage, tp, ps.ca, ps.oa);
                load_words<VPT, CW>(stb, L.off_in_stage, tp, ps.cb, ps.ob);
                ps.ob = hb ? ps.ob : ps.oa;
#pragma unroll
                for (int t = 0; t < VPT; ++t)
#pragma unroll
                    for (int c = 0; c < CW; ++c) ps.cb[t][c] = hb ? ps.cb[t][c] : 0u;
                float2 h2[2] = {make_float2(0.f, 0.f), make_float2(0.f, 0.f)};
#pragma unroll
                for (int t = 0; t < VPT; ++t) {
                    // padded views (k >= V) have zero A: no per-view branch
                    float2 fa[2], fb[2], fab[2];
                    avals(ps.ca[t], fa);
                    avals(ps.cb[t], fb);
                    const int oa = off_of(ps.oa, t), ob = off_of(ps.ob, t);
                    shifted<U8>(ps.ca[t][0], fa, ob - oa, fab);  // A_a on b's channels
                    const float* pw = sb_w + oa * VS + kv[t];
                    const float* qw = sb_w + ob * VS + kv[t];
                    ps.wa[t][0] = __fmul2_rn(make_float2(pw[0], pw[VS]), fa[0]);
                    ps.wa[t][1] = __fmul2_rn(make_float2(pw[2 * VS], pw[3 * VS]), fa[1]);
                    ps.wb[t][0] = __fmul2_rn(make_float2(qw[0], qw[VS]), fb[0]);
                    ps.wb[t][1] = __fmul2_rn(make_float2(qw[2 * VS], qw[3 * VS]), fb[1]);
                    h2[t & 1] = __ffma2_rn(ps.wb[t][0], fab[0], h2[t & 1]);
                    h2[t & 1] = __ffma2_rn(ps.wb[t][1], fab[1], h2[t & 1]);
                }
                // this lane's part of H; the warp reduction is done with the pair's theta1 sums
                const float2 hs = __fadd2_rn(h2[0], h2[1]);
                ps.hh = hs.x + hs.y;
            };
            // one voxel pair: theta1 partials from e -> barrier A -> the next pair's state ->
            // barrier B (deltas) -> scatter -> refill the next pair's stages
            auto pair_step = [&](int idx, PairState& cur, PairState& nxt) {
                const uint32_t pn = pseq + (uint32_t)(idx >> 1);  // running pair number
                if (lane == 0 && (vw == 0 || vw == 5)) stamp(idx >> 1, vw == 0 ? 0 : 8);
                const int buf = (int)(pn % kPairBufs);
                // ---- the pair's theta1 partials: sum (w A_a) e and sum (w A_b) e over this
                //      thread's views, from the state of e after the previous pair's scatter
                float2 ea[VPT][2], eb[VPT][2];
                {
                    float2 acc[2] = {make_float2(0.f, 0.f), make_float2(0.f, 0.f)};
                    float2 accb[2] = {acc[0], acc[0]};
#pragma unroll
                    for (int t = 0; t < VPT; ++t) {
                        const float* pe = sb_e + off_of(cur.oa, t) * VS + kv[t];
                        const float* qe = sb_e + off_of(cur.ob, t) * VS + kv[t];
                        ea[t][0] = make_float2(pe[0], pe[VS]);
                        ea[t][1] = make_float2(pe[2 * VS], pe[3 * VS]);
                        eb[t][0] = make_float2(qe[0], qe[VS]);
                        eb[t][1] = make_float2(qe[2 * VS], qe[3 * VS]);
                        acc[t & 1] = __ffma2_rn(cur.wa[t][0], ea[t][0], acc[t & 1]);
                        acc[t & 1] = __ffma2_rn(cur.wa[t][1], ea[t][1], acc[t & 1]);
                        accb[t & 1] = __ffma2_rn(cur.wb[t][0], eb[t][0], accb[t & 1]);
                        accb[t & 1] = __ffma2_rn(cur.wb[t][1], eb[t][1], accb[t & 1]);
                    }
                    const float2 ac = __fadd2_rn(acc[0], acc[1]), acb = __fadd2_rn(accb[0], accb[1]);
                    float2 gab = make_float2(ac.x + ac.y, acb.x + acb.y);
                    float hh = cur.hh;
#pragma unroll
                    for (int o = 16; o > 0; o >>= 1) {
                        const float2 r = make_float2(__shfl_xor_sync(kFull, gab.x, o), __shfl_xor_sync(kFull, gab.y, o));
                        hh += __shfl_xor_sync(kFull, hh, o);
                        gab = __fadd2_rn(gab, r);
                    }
                    if (lane == 0) {
                        float* rs = red + buf * 3 * NSL + gvw;
                        rs[0] = gab.x;
                        rs[NSL] = gab.y;
                        rs[2 * NSL] = hh;
                        if (CL == 2) {
                            // the same slots of the peer CTA, then arrive on both CTAs' pair
                            // barriers (the release orders the stores)
                            const uint32_t pa = peer_addr(rs, crank ^ 1u);
                            st_peer_f32(pa, gab.x);
                            st_peer_f32(pa + 4 * NSL, gab.y);
                            st_peer_f32(pa + 8 * NSL, hh);
                            mbar_arrive_peer(peer_addr(pairbar + buf, crank ^ 1u));
                            mbar_arrive(pairbar + buf);
                        }
                    }
                }
                // barrier A: arrive (the prior warp derives the deltas)
                if (lane == 0 && (vw == 0 || vw == 5)) stamp(idx >> 1, vw == 0 ? 1 : 9);
                if (CL == 1) asm volatile("bar.arrive 1, %0;" ::"r"(npair_threads) : "memory");
                // ---- meanwhile: the next pair's e-independent state
                nxt.sj = cur.sj + 2 >= R ? cur.sj + 2 - R : cur.sj + 2;
                if (idx + 2 < nact) prep(idx + 2, idx + 3 < nact, nxt);
                // the next pair's stages are consumed (prep has used its records): refill them
                // with the records R voxels ahead while the deltas are being derived (one commit
                // group per voxel, empty past the visit's end, keeps the wait counts fixed)
                {
                    const int s1 = nxt.sj + 1 == R ? 0 : nxt.sj + 1;
                    copy_record_to(idx + 2 + R, nxt.sj, nxt.lv[0]);
                    copy_record_to(idx + 3 + R, s1, nxt.lv[1]);
                }
                if (lane == 0 && (vw == 0 || vw == 5)) stamp(idx >> 1, vw == 0 ? 2 : 10);
                // ---- barrier B: the deltas are published
                {
                    const long long tw0 = (PROF && P.tprof) ? clock64() : 0;
                    asm volatile("bar.sync 2, %0;" ::"r"(npair_threads) : "memory");
                    if (lane == 0 && (vw == 0 || vw == 5)) stamp(idx >> 1, vw == 0 ? 3 : 11);
                    if (PROF && P.tprof && lane == 0)  // development aid: per-warp wait for the deltas
                        atomicAdd(P.tprof + 10 + warp, (unsigned long long)(clock64() - tw0));
                }
                // ---- Alg1:9-11 for both voxels on this thread's views: a's channels first with
                //      a's update, then b's channels with both updates -- b's path rewrites the
                //      entries the two voxels share with the full value, so A_b is never needed on
                //      a's channels
                const float sda = dslot[(pn & 1) * 2], sdb = dslot[(pn & 1) * 2 + 1];
                if (sda != 0.f || sdb != 0.f) {
                    const float2 nda = make_float2(-sda, -sda), ndb = make_float2(-sdb, -sdb);
                    auto put2 = [&](float* p, float2 v0, float2 v1) {
                        p[0] = v0.x;
                        p[VS] = v0.y;
                        p[2 * VS] = v1.x;
                        p[3 * VS] = v1.y;
                    };
#pragma unroll
                    for (int t = 0; t < VPT; ++t) {
                        float2 fa[2], fb[2], fab[2];
                        avals(cur.ca[t], fa);
                        avals(cur.cb[t], fb);
                        const int oa = off_of(cur.oa, t), ob = off_of(cur.ob, t);
                        shifted<U8>(cur.ca[t][0], fa, ob - oa, fab);
                        put2(sb_e + oa * VS + kv[t], __ffma2_rn(fa[0], nda, ea[t][0]), __ffma2_rn(fa[1], nda, ea[t][1]));
                        put2(sb_e + ob * VS + kv[t], __ffma2_rn(fb[0], ndb, __ffma2_rn(fab[0], nda, eb[t][0])),
                             __ffma2_rn(fb[1], ndb, __ffma2_rn(fab[1], nda, eb[t][1])));
                    }
                }
                if (lane == 0 && (vw == 0 || vw == 5)) stamp(idx >> 1, vw == 0 ? 4 : 12);
            };
            // the A records of the first R voxels (every stage is free: the previous visit ended
            // with a CTA-wide barrier), then the first pair's state; its stages are refilled.
            // The pair loop is unrolled by two so the two states swap roles without copies.
            PairState st0, st1;
            for (int i = 0; i < R; ++i) copy_record(i, tp);
            st0.sj = sbase;
            prep(0, 1 < nact, st0);
            copy_record(R, tp);
            copy_record(R + 1, tp);
            for (int idx = 0; idx < nact; idx += 4) {
                pair_step(idx, st0, st1);
                if (idx + 2 < nact) pair_step(idx + 2, st1, st0);
            }
        } else {
            // ---- prior warp: the surrogate terms of the first pair, then per pair: wait for the
            //      view warps' partial sums (A), derive both deltas (every lane, identical
            //      inputs), publish them (B), store the new values, next pair's surrogate terms
            prior_pair(tof, 0, nact, xt, cslot, TW, gx0, gy0, zg, P, nb, lane, pri + (pseq % kPairBufs));
            for (int idx = 0; idx < nact; idx += 2) {
                const uint32_t pn = pseq + (uint32_t)(idx >> 1);
                const int buf = (int)(pn % kPairBufs);
                const bool hasb = idx + 1 < nact;
                {
                    const long long tw0 = (PROF && P.tprof) ? clock64() : 0;
                    if (lane == 0) stamp(idx >> 1, 5);
                    if (CL == 1)
                        asm volatile("bar.sync 1, %0;" ::"r"(npair_threads) : "memory");
                    else
                        mbar_wait_cluster(pairbar + buf, (pn / kPairBufs) & 1u);
                    if (lane == 0) stamp(idx >> 1, 6);
                    if (PROF && P.tprof && lane == 0)  // development aid: wait for the partial sums
                        atomicAdd(P.tprof + 10 + warp, (unsigned long long)(clock64() - tw0));
                }
                const float* rb = red + buf * 3 * NSL;  // nvw <= NSL partials per quantity, rest 0
                const float sa = sum_slots<NSL>(rb), sbs = sum_slots<NSL>(rb + NSL), sh = sum_slots<NSL>(rb + 2 * NSL);
                const PriPair pp = pri[buf];
                const float scale_a = vscale[idx];
                float ua = pp.va;
                const float theta1a = -scale_a * sa;  // Alg1:5
                const float theta2a = vth2[idx];      // Alg1:6 (precomputed)
                {
                    const float num = theta2a * pp.va - theta1a + 2.f * pp.sxa;
                    const float den = theta2a + 2.f * pp.sa;
                    if (den > 0.f) ua = __fdividef(num, den);
                    if (P.pc.positivity) ua = fmaxf(ua, 0.f);
                }
                const float da = ua - pp.va;  // Alg1:7-8
                float ub = pp.vb, db = 0.f, scale_b = 0.f, theta1b = 0.f, theta2b = 0.f;
                if (hasb) {
                    scale_b = vscale[idx + 1];
                    // e after a's update: sum w A_b e' = s_b (S_b - s_a delta_a H)
                    const float theta1 = theta1b = -scale_b * fmaf(-scale_a * da, sh, sbs);
                    const float theta2 = theta2b = vth2[idx + 1];
                    float psb = pp.sb, psx = pp.sxb;
                    if (pp.bab != 0.f) {  // a is b's neighbour: its term with a's new value
                        const float bn = pp.bab * phi_f(P.pc, pp.vb - ua);
                        psb += bn - pp.btab;
                        psx += bn * ua - pp.btab * pp.va;
                    }
                    const float num = theta2 * pp.vb - theta1 + 2.f * psx;
                    const float den = theta2 + 2.f * psb;
                    if (den > 0.f) ub = __fdividef(num, den);
                    if (P.pc.positivity) ub = fmaxf(ub, 0.f);
                    db = ub - pp.vb;
                }
                if (lane == 0) {
                    dslot[(pn & 1) * 2] = scale_a * da;
                    dslot[(pn & 1) * 2 + 1] = scale_b * db;
                }
                if (P.dump && lane == 0) {
                    // test hook (mbir_set_update_dump): the pair's (voxel, theta1, theta2, delta)
                    // exactly as the delta chain used them (b's theta1 includes a's update), a then b
                    const unsigned long long slot = atomicAdd(P.dump_count, hasb ? 2ull : 1ull);
                    for (int u = 0; u < (hasb ? 2 : 1); ++u) {
                        const int tv = tof[idx + u];
                        const uint32_t vox = (uint32_t)(((size_t)z * P.ny + gy0 + (tv >> 8)) * P.nx + gx0 + (tv & 255));
                        if (slot + u < (unsigned long long)P.dump_cap)
                            *(float4*)(P.dump + 4 * (slot + u)) = make_float4(
                                __uint_as_float(vox), u ? theta1b : theta1a, u ? theta2b : theta2a, u ? db : da);
                    }
                }
                if (lane == 0) stamp(idx >> 1, 7);
                asm volatile("bar.arrive 2, %0;" ::"r"(npair_threads) : "memory");  // barrier B
                // the pair's new values, then the next pair's surrogate terms
                if (lane == 0) {
                    const int ta = tof[idx];
                    xt[cslot + (ta >> 8) * TW + (ta & 255)] = ua;
                    if (hasb) {
                        const int tbv = tof[idx + 1];
                        xt[cslot + (tbv >> 8) * TW + (tbv & 255)] = ub;
                    }
                    amount += fabsf(da) + fabsf(db);
                }
                __syncwarp();
                const long long tr0 = (PROF && P.tprof) ? clock64() : 0;
                if (idx + 2 < nact)
                    prior_pair(tof, idx + 2, nact, xt, cslot, TW, gx0, gy0, zg, P, nb, lane,
                               pri + (pn + 1) % kPairBufs);
                if (PROF && P.tprof && lane == 0) atomicAdd(P.tprof + 24, (unsigned long long)(clock64() - tr0));
                if (lane == 0) stamp(idx >> 1, 13);
            }
        }
        gseq += nact;
        pseq += (uint32_t)(nact + 1) >> 1;
        ++ntask;
        if (PROF && P.tprof && threadIdx.x == 0) tp3 = clock64();
        if (threadIdx.x == 0) stamp(60, 3);
        __syncthreads();

        // ---- 6. write-back: delta e of the band, atomically, and the SV's voxels
        if (is_view) {
            float* ez = P.e + (size_t)z * V * M;
            // the final band goes back through the staging tile (stride 33, as in the pack), then
            // each aligned 32-float row window gets delta = final - e_init (band positions only)
            // with red.global.add.v4.f32
            const int sub = lane >> 3, ch = lane & 7;
            // e_init windows of tile t (L2-resident scratch), one tile ahead of the staging
            auto ld_init = [&](int t, float4 (&s4)[8]) {
                const int k0 = (vw * VPT + t) * 32;
#pragma unroll
                for (int m = 0; m < 8; ++m) s4[m] = __ldcg((const float4*)(scr + (k0 + 4 * m + sub) * 32 + 4 * ch));
            };
            float4 s4b[2][8];
            ld_init(0, s4b[0]);
#pragma unroll
            for (int t = 0; t < VPT; ++t) {
                if (t + 1 < VPT) ld_init(t + 1, s4b[(t + 1) & 1]);
                const float4 (&s4)[8] = s4b[t & 1];
                const int k0 = (vw * VPT + t) * 32;
                const int kk = k0 + lane;
                const uint32_t bi = vbase + kk < V ? binfo[tb * VL + kk] : 0u;
                const int bw = (int)(bi & 31u), roff = (int)(bi >> 5);
                const uint32_t bmask = ((1u << bw) - 1u) << (roff & 3);
                // this view's final band -> its staging row (positions outside the band: 0)
                const float* se = sb_e + kk - (roff & 3) * VS;
#pragma unroll
                for (int q4 = 0; q4 < 8; ++q4) {
                    float rv[4];
#pragma unroll
                    for (int j = 0; j < 4; ++j) {
                        const int p = 4 * q4 + j;
                        rv[j] = (bmask & (1u << p)) ? se[p * VS] : 0.f;
                    }
                    *(float4*)(stg_w + lane * kStg + 4 * q4) = make_float4(rv[0], rv[1], rv[2], rv[3]);
                }
                __syncwarp();
#pragma unroll
                for (int m = 0; m < 8; ++m) {
                    const int i = 4 * m + sub;
                    const int oi = __shfl_sync(kFull, roff, i);
                    const uint32_t nib = __shfl_sync(kFull, bmask, i) >> (4 * ch);
                    const int s = oi & 3;
                    const float4 f4 = *(const float4*)(stg_w + i * kStg + 4 * ch);
                    const float fv[4] = {f4.x, f4.y, f4.z, f4.w};
                    float d[4];
                    const float e0[4] = {s4[m].x, s4[m].y, s4[m].z, s4[m].w};
#pragma unroll
                    for (int j = 0; j < 4; ++j) d[j] = (nib & (1u << j)) ? fv[j] - e0[j] : 0.f;
                    if (vbase + k0 + i < V && (d[0] != 0.f || d[1] != 0.f || d[2] != 0.f || d[3] != 0.f))
                        red_add_v4(ez + (oi - s) + 4 * ch, d[0], d[1], d[2], d[3]);
                }
                __syncwarp();
            }
        } else {
            // prior warp: the image and the counters (rank 0 only), then the next task's band
            // info with an L2 warm-up of its band rows (the next pack then reads L2)
            if (crank == 0) {
                for (int i = lane; i < tw * th; i += 32) {
                    const int lx = i % tw, ly = i / tw;
                    P.x[(size_t)(z + 1) * plane + (size_t)(gy0 + ly) * P.nx + gx0 + lx] =
                        xt[cslot + ly * TW + lx];
                }
                if (lane == 0) {
                    P.sv_amount[(size_t)z * P.nsv + sv] = amount;
                    atomicAdd(P.counters + 0, (unsigned long long)nact);
                    atomicAdd(P.counters + 1, (unsigned long long)(tw * th - nact));
                    atomicAdd(P.counters + 2, 1ull);
                    atomicAdd(P.sum_delta, (double)amount);
                }
            } else if (lane == 0) {
                mbar_wait_cluster(taskbar, (ntask - 1u) & 1u);  // rank 0 published the next task
            }
            __syncwarp();
            const int nq = s_task[nslot];
            if (nq < tend) {
                const int nt = P.flat[nq];
                constexpr int KMAX = 12;  // views per lane and pass: all loads in flight at once
                const int psv = nt & 16383, pz = nt >> 14;
                uint32_t* dst = binfo + (tb ^ 1) * VL - vbase;  // indexed by task view k
                const int kend = min(V, vbase + VL);
                const float* wz = P.w + (size_t)pz * V * M;
                const float* ez = P.e + (size_t)pz * V * M;
#pragma unroll 1
                for (int k0 = vbase; k0 < kend; k0 += 32 * KMAX) {
                    int bs[KMAX], bwd[KMAX];
#pragma unroll
                    for (int i = 0; i < KMAX; ++i) {
                        const int k = k0 + lane + 32 * i;
                        if (k < kend) {
                            bs[i] = P.A.band_start[(size_t)psv * V + k];
                            bwd[i] = P.A.band_width[(size_t)psv * V + k];
                        }
                    }
#pragma unroll
                    for (int i = 0; i < KMAX; ++i) {
                        const int k = k0 + lane + 32 * i;
                        if (k < kend) {
                            const int r = k * M + bs[i], r1 = r + max(bwd[i], 1) - 1;
                            dst[k] = ((uint32_t)r << 5) | (uint32_t)bwd[i];
                            asm volatile("prefetch.global.L2 [%0];" ::"l"(wz + r));
                            asm volatile("prefetch.global.L2 [%0];" ::"l"(wz + r1));
                            asm volatile("prefetch.global.L2 [%0];" ::"l"(ez + r));
                            asm volatile("prefetch.global.L2 [%0];" ::"l"(ez + r1));
                        }
                    }
                }
            }
        }
        if (CL == 2) cluster_sync_all(); else __syncthreads();
        if (threadIdx.x == 0) {
            stamp(60, 4);
            if (TR) P.trace[0] = 1ull + (unsigned long long)nact;
        }
        if (PROF && P.tprof && threadIdx.x == 0 && crank == 0) {
            const long long tp4 = clock64();
            atomicAdd(P.tprof + 0, (unsigned long long)(tp1 - tp0));  // x tile, zero-skip, order
            atomicAdd(P.tprof + 1, (unsigned long long)(tp2 - tp1));  // SVB pack (+ first A stage)
            atomicAdd(P.tprof + 2, (unsigned long long)(tp3 - tp2));  // voxel loop
            atomicAdd(P.tprof + 3, (unsigned long long)(tp4 - tp3));  // write-back
            atomicAdd(P.tprof + 4, (unsigned long long)nact);
            atomicAdd(P.tprof + 5, 1ull);
            atomicAdd(P.tprof + 6, (unsigned long long)(tp1b - tp1));  // view-warp 0's own pack
        }
    }
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

// A-record ring depth (voxels of cp.async lookahead): u8 records are 5 B/view, fp32 ones 17 B/view
// (the pair loop needs >= 4: the current pair's two stages plus the next pair's two).  The
// cluster variant holds half a record per stage but must fit two CTAs per SM.
constexpr int ring_depth(bool u8, int cl) { return u8 ? (cl == 2 ? 8 : 12) : 4; }

int icd_smem_bytes(const IcdParams& p, int vpt, int nnb, bool quantize, int cl)
{
    return smem_layout(p.rows, svb_stride(vpt, cl), p.side, p.S2, nnb, p.A.VA, quantize,
                       ring_depth(quantize, cl), p.nvw, cl).total;
}

template <int VPT, bool U8, int NNB, int CL>
static cudaError_t launch_icd_t(const IcdParams& p, int gx, int gy, cudaStream_t st)
{
    constexpr int R = ring_depth(U8, CL);
    // the phase-profiling instrumentation (env MBIR_PHASE_PROFILE) is compiled only into the
    // bench's configuration; every other launch runs the instrumentation-free kernel
    constexpr bool kProfiled = VPT == 4 && U8 && CL == 1;
    auto kern = (kProfiled && (p.tprof || p.trace)) ? k_icd_sv<VPT, U8, NNB, R, CL, kProfiled> : k_icd_sv<VPT, U8, NNB, R, CL, false>;
    IcdParams q = p;
    q.lay = smem_layout(p.rows, svb_stride(VPT, CL), p.side, p.S2, NNB, p.A.VA, U8, R, p.nvw, CL);
    const int smem = q.lay.total;
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    if (e != cudaSuccess) return e;
    e = cudaFuncSetAttribute(kern, cudaFuncAttributePreferredSharedMemoryCarveout, 100);
    if (e != cudaSuccess) return e;
    const int threads = 32 * (p.nvw / CL + 1);  // view warps + prior warp
    if (CL == 1) {
        kern<<<dim3(gx, gy), threads, smem, st>>>(q);
        return cudaGetLastError();
    }
    cudaLaunchConfig_t cfg{};
    cfg.gridDim = dim3(gx, gy);
    cfg.blockDim = dim3(threads);
    cfg.dynamicSmemBytes = smem;
    cfg.stream = st;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeClusterDimension;
    at[0].val.clusterDim.x = CL;
    at[0].val.clusterDim.y = 1;
    at[0].val.clusterDim.z = 1;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    return cudaLaunchKernelEx(&cfg, kern, q);
}

// resident CTAs of the update kernel per device (occupancy query; clusters x CL for CL = 2)
template <int VPT, bool U8, int NNB, int CL>
static int resident_ctas_t(const IcdParams& p)
{
    constexpr int R = ring_depth(U8, CL);
    auto kern = k_icd_sv<VPT, U8, NNB, R, CL, false>;
    const int smem = smem_layout(p.rows, svb_stride(VPT, CL), p.side, p.S2, NNB, p.A.VA, U8, R, p.nvw, CL).total;
    if (cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, smem) != cudaSuccess) return -1;
    cudaFuncSetAttribute(kern, cudaFuncAttributePreferredSharedMemoryCarveout, 100);
    const int threads = 32 * (p.nvw / CL + 1);
    if (getenv("MBIR_OCC_DEBUG")) {
        int nb = -1;
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, kern, threads, smem);
        cudaFuncAttributes fa{};
        cudaFuncGetAttributes(&fa, kern);
        fprintf(stderr, "[mbir occ] CL %d threads %d smem %d blocks/SM (no cluster) %d regs %d static smem %zu local %zu\n",
                CL, threads, smem, nb, fa.numRegs, fa.sharedSizeBytes, fa.localSizeBytes);
    }
    if (CL == 1) {
        int nb = 0;
        if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, kern, threads, smem) != cudaSuccess) return -1;
        int dev = 0, nsm = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
        return nb * nsm;
    }
    cudaLaunchConfig_t cfg{};
    cfg.gridDim = dim3(2 * 148);
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

int icd_resident_ctas(const IcdParams& p, int vpt, int nnb, bool quantize, int cl)
{
    if (vpt == 1) {
        if (quantize) return nnb == 26 ? resident_ctas_t<1, true, 26, 1>(p) : resident_ctas_t<1, true, 8, 1>(p);
        return nnb == 26 ? resident_ctas_t<1, false, 26, 1>(p) : resident_ctas_t<1, false, 8, 1>(p);
    }
    if (quantize && cl == 2 && vpt == 2) return nnb == 26 ? resident_ctas_t<2, true, 26, 2>(p) : resident_ctas_t<2, true, 8, 2>(p);
    if (quantize && cl == 2) return nnb == 26 ? resident_ctas_t<4, true, 26, 2>(p) : resident_ctas_t<4, true, 8, 2>(p);
    if (quantize) return nnb == 26 ? resident_ctas_t<4, true, 26, 1>(p) : resident_ctas_t<4, true, 8, 1>(p);
    return nnb == 26 ? resident_ctas_t<4, false, 26, 1>(p) : resident_ctas_t<4, false, 8, 1>(p);
}

cudaError_t launch_icd(const IcdParams& p, int vpt, int nnb, bool quantize, int cl, int gx, int gy,
                       cudaStream_t st)
{
    if (vpt == 1) {
        if (quantize) return nnb == 26 ? launch_icd_t<1, true, 26, 1>(p, gx, gy, st) : launch_icd_t<1, true, 8, 1>(p, gx, gy, st);
        return nnb == 26 ? launch_icd_t<1, false, 26, 1>(p, gx, gy, st) : launch_icd_t<1, false, 8, 1>(p, gx, gy, st);
    }
    if (quantize && cl == 2 && vpt == 2)
        return nnb == 26 ? launch_icd_t<2, true, 26, 2>(p, gx, gy, st) : launch_icd_t<2, true, 8, 2>(p, gx, gy, st);
    if (quantize && cl == 2)
        return nnb == 26 ? launch_icd_t<4, true, 26, 2>(p, gx, gy, st) : launch_icd_t<4, true, 8, 2>(p, gx, gy, st);
    if (quantize) return nnb == 26 ? launch_icd_t<4, true, 26, 1>(p, gx, gy, st) : launch_icd_t<4, true, 8, 1>(p, gx, gy, st);
    return nnb == 26 ? launch_icd_t<4, false, 26, 1>(p, gx, gy, st) : launch_icd_t<4, false, 8, 1>(p, gx, gy, st);
}

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
