// libmbir C-ABI (include/mbir.h): handle lifecycle, host orchestration of Alg. 3,
// the z-slab multi-GPU halo exchange over NCCL, and the test hooks.
//
// Host loop per iteration (Alg3:16-31):
//   select (device: all / top 25 % / random 25 %, 4 checkerboard colours per slice)
//   for z-parity half (3-D prior only): for colour 0..3: for batch: fused update kernel
//   [multi-GPU] after each half: NCCL send/recv of the updated boundary slices (halo)
//   counters -> equits, all-reduced across ranks
#include <dlfcn.h>
#include <math.h>
#include <nccl.h>
#include <stdio.h>
#include <string.h>

#include <algorithm>
#include <condition_variable>
#include <mutex>
#include <new>
#include <string>
#include <vector>

#include "mbir_internal.h"

using namespace mbir;

// views per lane of the update kernel for > 128 views (build-time choice: 4 = six view warps,
// 2 = twelve)

namespace {

// ---- NCCL through dlopen (only needed when nranks > 1) ----
struct NcclApi {
    bool ok = false;
    ncclResult_t (*GetUniqueId)(ncclUniqueId*) = nullptr;
    ncclResult_t (*CommInitRank)(ncclComm_t*, int, ncclUniqueId, int) = nullptr;
    ncclResult_t (*CommDestroy)(ncclComm_t) = nullptr;
    ncclResult_t (*Send)(const void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
    ncclResult_t (*Recv)(void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
    ncclResult_t (*AllReduce)(const void*, void*, size_t, ncclDataType_t, ncclRedOp_t, ncclComm_t,
                              cudaStream_t) = nullptr;
    ncclResult_t (*GroupStart)() = nullptr;
    ncclResult_t (*GroupEnd)() = nullptr;
    const char* (*GetErrorString)(ncclResult_t) = nullptr;
};

NcclApi& nccl()
{
    static NcclApi api;
    static bool tried = false;
    if (tried) return api;
    tried = true;
    void* lib = dlopen("libnccl.so.2", RTLD_NOW | RTLD_NOLOAD);
    if (!lib) lib = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
    if (!lib) lib = dlopen("libnccl.so", RTLD_NOW | RTLD_GLOBAL);
    if (!lib) return api;
#define LOADSYM(f) api.f = (decltype(api.f))dlsym(lib, "nccl" #f)
    LOADSYM(GetUniqueId);
    LOADSYM(CommInitRank);
    LOADSYM(CommDestroy);
    LOADSYM(Send);
    LOADSYM(Recv);
    LOADSYM(AllReduce);
    LOADSYM(GroupStart);
    LOADSYM(GroupEnd);
    LOADSYM(GetErrorString);
#undef LOADSYM
    api.ok = api.GetUniqueId && api.CommInitRank && api.CommDestroy && api.Send && api.Recv &&
             api.AllReduce && api.GroupStart && api.GroupEnd;
    return api;
}

}  // namespace

struct mbir_handle;

// Test hook (mbir_link_slabs): handles owning consecutive slabs of one volume on ONE device,
// exchanging halo slices by device-to-device copies behind a host barrier instead of NCCL.
struct LocalGroup {
    std::mutex mu;
    std::condition_variable cv;
    int n = 0, arrived = 0;
    unsigned long long generation = 0;
    std::vector<mbir_handle*> members;  // by rank
    void barrier()
    {
        std::unique_lock<std::mutex> lk(mu);
        const unsigned long long gen = generation;
        if (++arrived == n) {
            arrived = 0;
            ++generation;
            cv.notify_all();
        } else {
            cv.wait(lk, [&] { return generation != gen; });
        }
    }
};

struct mbir_handle {
    mbir_geometry g{};
    std::vector<double> angles;
    mbir_prior pr{};
    mbir_options o{};
    int device = 0;
    cudaStream_t st = nullptr;
    bool own_stream = false;
    int rank = 0, nranks = 1;
    ncclComm_t comm = nullptr;
    LocalGroup* lg = nullptr;  // mbir_link_slabs group (shared by its members; rank 0 frees it)
    int side = 0, nsvx = 0, nsvy = 0, nsv = 0, S2 = 0, nsv_pad = 0;
    int rows = 0, band_max = 0, nwin = 1;
    int vpt = 1, nvw = 0, Vs = 0, threads = 0, smem = 0, blocks_per_sm = 1, nsm = 148;
    int cl = 1;  // update-kernel CTAs per SV task (2: thread-block cluster splitting the views)
    int kv = 1;  // voxels per step of the update kernel (2: voxel pairs)
    int resident = 0;  // update-kernel CTAs resident on the device at once (occupancy query)
    int max_group = 0;
    DevA A{};
    double* d_cs = nullptr;
    float *d_y = nullptr, *d_w = nullptr, *d_e = nullptr, *d_x = nullptr;
    float *d_theta2 = nullptr, *d_amount = nullptr, *d_scratch = nullptr;
    uint8_t* d_perm = nullptr;  // [kNPerm][S2] voxel visiting orders
    static constexpr int kNPerm = 64;
    int *d_task_list = nullptr, *d_task_count = nullptr;
    int *d_flat = nullptr, *d_brange = nullptr, *d_fetch = nullptr;
    unsigned int* d_gbar = nullptr;  // [8 phases] grid-barrier counters of the update kernel
    int* d_keep = nullptr;  // zero-skip pre-filter flags of the current phase list
    unsigned long long* d_counters = nullptr;  // [updates, skipped, visits, empty visits]
    double* d_sum_delta = nullptr;
    int* d_flag = nullptr;
    double* d_acc = nullptr;
    unsigned long long* h_counters = nullptr;  // pinned [5] (4 counters + sum_delta bits)
    bool have_sino = false;
    bool theta2_ok = false;  // d_theta2 holds sum w A^2 for the current weights
    bool x_zero = true;  // the image is known to be all zero (then e = y needs no projection)
    int iter = 0;
    int64_t nnz = 0, a_bytes = 0, band_entries = 0;
    cudaEvent_t ev0 = nullptr, ev1 = nullptr;
    std::vector<cudaEvent_t> kev;  // per-launch event pairs of the update kernel (one iteration)
    int kev_used = 0;
    unsigned long long* d_tprof = nullptr;  // phase cycle counters (env MBIR_PHASE_PROFILE)
    PriorConst pc{};  // q-GGMRF constants and neighbourhood, passed to every kernel by value
    // per-update record (test hook mbir_set_update_dump): [cap][4] = (voxel, theta1, theta2, delta)
    float* d_dump = nullptr;
    unsigned long long* d_dump_count = nullptr;
    int64_t dump_cap = 0;
    std::string err;
};

namespace {

int fail(mbir_handle* h, int code, const std::string& msg)
{
    if (h) h->err = msg;
    return code;
}

#define CK(call)                                                                             \
    do {                                                                                     \
        cudaError_t e_ = (call);                                                             \
        if (e_ != cudaSuccess)                                                               \
            return fail(h, e_ == cudaErrorMemoryAllocation ? MBIR_ENOMEM : MBIR_ECUDA,       \
                        std::string(#call) + ": " + cudaGetErrorString(e_));                 \
    } while (0)

#define CKN(call)                                                                            \
    do {                                                                                     \
        ncclResult_t r_ = (call);                                                            \
        if (r_ != ncclSuccess)                                                               \
            return fail(h, MBIR_ENCCL, std::string(#call) + ": " +                           \
                               (nccl().GetErrorString ? nccl().GetErrorString(r_) : "nccl error")); \
    } while (0)

IcdParams make_params(mbir_handle* h)
{
    IcdParams p{};
    p.nx = h->g.nx;
    p.ny = h->g.ny;
    p.nz_local = h->g.nz_local;
    p.z_offset = h->g.z_offset;
    p.nz_total = h->g.nz_total;
    p.V = h->g.nviews;
    p.M = h->g.nchannels;
    p.side = h->side;
    p.nsvx = h->nsvx;
    p.nsv = h->nsv;
    p.S2 = h->S2;
    p.Vs = h->Vs;
    p.rows = h->rows;
    p.nwin = h->nwin;
    p.nvw = h->nvw;
    p.nbatch = 1;
    p.gbar = h->d_gbar;
    p.A = h->A;
    p.e = h->d_e;
    p.w = h->d_w;
    p.x = h->d_x;
    p.theta2 = h->d_theta2;
    p.scratch = h->d_scratch;
    p.perm = h->d_perm;
    p.nperm = mbir_handle::kNPerm;
    p.sv_amount = h->d_amount;
    p.counters = h->d_counters;
    p.sum_delta = h->d_sum_delta;
    p.seed = h->o.seed;
    p.iter = h->iter;
    p.deterministic = h->o.deterministic;
    p.kv = h->kv;
    p.tprof = h->d_tprof;
    p.pc = h->pc;
    p.dump = h->d_dump;
    p.dump_count = h->d_dump_count;
    p.dump_cap = h->dump_cap;
    return p;
}

size_t sino_elems(const mbir_handle* h)
{
    return (size_t)h->g.nz_local * h->g.nviews * h->g.nchannels;
}
size_t plane_elems(const mbir_handle* h) { return (size_t)h->g.nx * h->g.ny; }

cudaMemcpyKind kind_in(int where) { return where == MBIR_DEVICE ? cudaMemcpyDeviceToDevice : cudaMemcpyHostToDevice; }
cudaMemcpyKind kind_out(int where) { return where == MBIR_DEVICE ? cudaMemcpyDeviceToDevice : cudaMemcpyDeviceToHost; }

// halo exchange of the boundary slices whose global parity is `parity` (-1: both ends).
int exchange_halo(mbir_handle* h, int parity)
{
    if (h->nranks <= 1) return MBIR_OK;
    const size_t pl = plane_elems(h);
    int32_t ops[4][3];
    const int n = mbir_halo_plan(h->g.z_offset, h->g.nz_local, h->rank, h->nranks, parity, &ops[0][0]);
    if (n < 0) return fail(h, MBIR_EINVAL, "bad halo plan");
    if (!h->comm) {
        // linked slabs on one device (test hook): every member has finished the half (stream
        // synchronised) when the barrier opens; each then copies the peers' boundary slices it
        // receives into its halo.  The next half only writes slices of the other parity, and the
        // member cannot reach the next exchange before this copy completed, so one barrier per
        // exchange orders everything.
        if (!h->lg) return fail(h, MBIR_ESTATE, "nranks > 1 without NCCL: call mbir_link_slabs first");
        CK(cudaStreamSynchronize(h->st));
        h->lg->barrier();
        for (int i = 0; i < n; ++i) {
            if (ops[i][1]) continue;  // sends are the peer's receives
            const mbir_handle* p = h->lg->members[ops[i][0]];
            // my lower halo (0) <- the peer's last slice; my upper halo (nz + 1) <- its first
            const int src = ops[i][2] == 0 ? p->g.nz_local : 1;
            CK(cudaMemcpyAsync(h->d_x + (size_t)ops[i][2] * pl, p->d_x + (size_t)src * pl, pl * 4,
                               cudaMemcpyDeviceToDevice, h->st));
        }
        CK(cudaStreamSynchronize(h->st));
        h->lg->barrier();
        return MBIR_OK;
    }
    NcclApi& N = nccl();
    CKN(N.GroupStart());
    for (int i = 0; i < n; ++i) {
        float* buf = h->d_x + (size_t)ops[i][2] * pl;
        if (ops[i][1])
            CKN(N.Send(buf, pl, ncclFloat, ops[i][0], h->comm, h->st));
        else
            CKN(N.Recv(buf, pl, ncclFloat, ops[i][0], h->comm, h->st));
    }
    CKN(N.GroupEnd());
    return MBIR_OK;
}

// CUDA event pair around a run of update-kernel launches on the handle's stream (the batches of
// one phase: only batch-boundary gaps fall inside it; one pair per phase keeps the per-launch host
// work low for many-batch 2-D iterations)
int kev_mark(mbir_handle* h, bool begin)
{
    if (begin && (int)h->kev.size() < 2 * (h->kev_used + 1)) {
        for (int i = 0; i < 2; ++i) {
            cudaEvent_t e;
            CK(cudaEventCreate(&e));
            h->kev.push_back(e);
        }
    }
    CK(cudaEventRecord(h->kev[2 * h->kev_used + (begin ? 0 : 1)], h->st));
    if (!begin) h->kev_used++;
    return MBIR_OK;
}

// e = y - A x
int refresh_error(mbir_handle* h)
{
    IcdParams p = make_params(h);
    const bool q = h->o.quantize_A != 0;
    if (h->x_zero)  // e = y - A 0
        CK(cudaMemcpyAsync(h->d_e, h->d_y, sino_elems(h) * 4, cudaMemcpyDeviceToDevice, h->st));
    else
        CK(launch_forward(p, q, h->d_y, h->st));
    return MBIR_OK;
}

int run_iterations(mbir_handle* h, int n_iter, double target_equits, mbir_stats* st)
{
    if (!h->have_sino) return fail(h, MBIR_ESTATE, "mbir_set_sinogram has not been called");
    const double nvox_total = (double)h->g.nx * h->g.ny * h->g.nz_total;
    const bool q = h->o.quantize_A != 0;
    const int nnb = h->pr.neighborhood;
    const int parities = (nnb == 26 && h->g.nz_total > 1) ? 2 : 1;
    const int target_ctas = h->resident;  // persistent grid: every resident CTA (cluster)
    int64_t updates = 0, skipped = 0, visits = 0, empty = 0, iters = 0, launches = 0, klaunches = 0;
    int zero_iters = 0;  // consecutive iterations without an executed update
    double ksec = 0.0;
    double sum_delta = 0.0;
    CK(cudaEventRecord(h->ev0, h->st));
    for (int it = 0;; ++it) {
        if (n_iter >= 0 && it >= n_iter) break;
        if (n_iter < 0 && (double)updates >= target_equits * nvox_total) break;
        h->iter += 1;
        h->x_zero = false;
        h->kev_used = 0;
        CK(cudaMemsetAsync(h->d_counters, 0, 4 * sizeof(unsigned long long), h->st));
        CK(cudaMemsetAsync(h->d_sum_delta, 0, sizeof(double), h->st));
        // ---- SV selection (Alg3:17-23)
        SchedParams sp{};
        sp.nz_local = h->g.nz_local;
        sp.z_offset = h->g.z_offset;
        sp.nsvx = h->nsvx;
        sp.nsvy = h->nsvy;
        sp.nsv = h->nsv;
        sp.nsv_pad = h->nsv_pad;
        sp.max_group = h->max_group;
        sp.seed = h->o.seed;
        sp.iter = h->iter;
        sp.sv_amount = h->d_amount;
        sp.task_list = h->d_task_list;
        sp.task_count = h->d_task_count;
        // zero-skip re-admission iteration (reading R9): no zero-skipping, and a RANDOM subset, so
        // that SVs frozen at 0 (update amount 0, never among the "top" ones) are re-examined
        // (iterations 1 + k P, k >= 1: with an even period these are random-subset iterations
        // anyway, so the top-amount iterations stay as Alg. 3 has them)
        const bool readmit = h->o.zero_skip && h->o.zero_skip_period > 0 && h->iter > 1 &&
                             h->iter % h->o.zero_skip_period == 1 % h->o.zero_skip_period;
        if (h->o.deterministic) {
            sp.mode = 3;
            sp.nsel = h->nsv;
        } else if (h->iter == 1) {
            sp.mode = 0;
            sp.nsel = h->nsv;
        } else {
            sp.mode = (h->iter % 2 == 0 && !readmit) ? 1 : 2;
            sp.nsel = std::min(h->nsv, std::max(1, (int)ceil(h->o.sv_fraction * h->nsv - 1e-9)));
        }
        CK(launch_select(sp, h->st));
        ++launches;
        // ---- flat task lists + batch ranges per (z-parity, colour) phase (Alg3:24-27)
        const bool det = h->o.deterministic != 0;
        // batch_svs = 0 (auto): a whole colour group per launch, unless the phase has so few slices
        // that more than `cap` SVs of one slice would run at once -- then batches of `cap` SVs per
        // slice, each launch seeing the previous one's write-backs.  Same-colour SVs updated
        // concurrently fit the same residual along shared rays, and too many of them make
        // asynchronous SV-ICD oscillate or diverge (reading R22: on the paper's 512^2
        // geometry 42 per slice converge, 84 diverge; on 256^2 side-5 cases 39 oscillate, 20
        // converge).  cap = N / 12 SVs per slice of width N pixels, whatever the SV side.
        const int slices_in_phase = std::max(1, h->g.nz_local / parities);
        const int ray_cap = std::max(kAutoCapMin, (std::max(h->g.nx, h->g.ny) + kAutoCapDiv / 2) / kAutoCapDiv);
        const bool auto_batch = !det && h->o.batch_svs == 0 && target_ctas / h->cl > ray_cap * slices_in_phase;
        const int B = auto_batch ? ray_cap : (det || h->o.batch_svs <= 0) ? h->max_group : h->o.batch_svs;
        const int thr = (det || h->o.batch_svs <= 0) ? 0 : (h->o.batch_threshold >= 0 ? h->o.batch_threshold : B / 4);
        const int nb = (h->max_group + B - 1) / B;
        CK(launch_flatten(h->d_task_list, h->d_task_count, h->g.nz_local, h->g.z_offset, parities,
                          h->max_group, B, thr, nb, h->d_flat, h->d_brange, h->st));
        ++launches;
        CK(cudaMemsetAsync(h->d_fetch, 0, sizeof(int) * 8 * nb, h->st));
        CK(cudaMemsetAsync(h->d_gbar, 0, sizeof(unsigned int) * 8, h->st));
        IcdParams p = make_params(h);
        // theta2 = sum w A^2 (Alg1:6) after new weights: reduced inside the update kernel during an
        // iteration that visits every voxel (the first one, unless a batch threshold drops tasks);
        // otherwise by the separate k_theta2 pass first
        p.theta2_pass = 0;
        if (!h->theta2_ok) {
            if (h->iter == 1 && thr == 0) {
                p.theta2_pass = 1;
            } else {
                CK(launch_theta2(p, q, h->st));
                ++launches;
                h->theta2_ok = true;
            }
        }
        // zero-skip from iteration 2 on, except in re-admission iterations
        p.zero_skip_active = (h->o.zero_skip && h->iter > 1 && !readmit) ? 1 : 0;
        const size_t cap = (size_t)h->g.nz_local * h->max_group;
        // deterministic: one CTA (or one cluster) walks the phase list in order (sequential ICD,
        // known order)
        const int grid = det ? h->cl : target_ctas;
        // iterations >= 2 without batching: the tasks whose whole tile is zero are flagged per
        // phase (sched.cu k_zero_flags) and skipped at task fetch by the update kernel
        const bool prefilter = p.zero_skip_active && nb == 1 && !det;
        for (int zp = 0; zp < parities; ++zp) {
            for (int colour = 0; colour < 4; ++colour) {
                const int ph = zp * 4 + colour;
                p.flat = h->d_flat + ph * cap;
                p.keep = nullptr;
                if (prefilter) {
                    CK(launch_zero_flags(h->d_flat + ph * cap, h->d_brange + ph * (nb + 1), h->d_x, h->g.nx,
                                         h->g.ny, h->g.nz_local, h->g.z_offset, h->g.nz_total, h->side, h->nsvx,
                                         nnb, (int)cap, h->d_keep, h->st));
                    ++launches;
                    p.keep = h->d_keep;
                }
                if (int r = kev_mark(h, true)) return r;
                if (h->cl == 1 && h->kv == 1 && nb > 1) {
                    // one cooperative launch runs the phase's batches with grid barriers between
                    p.brange = h->d_brange + ph * (nb + 1);
                    p.fetch = h->d_fetch + ph * nb;
                    p.nbatch = nb;
                    p.gbar = h->d_gbar + ph;
                    CK(launch_svicd(p, h->vpt, nnb, q, h->cl, grid, h->st));
                    ++launches;
                    ++klaunches;
                } else {
                    for (int b = 0; b < nb; ++b) {
                        p.brange = h->d_brange + ph * (nb + 1) + b;
                        p.fetch = h->d_fetch + ph * nb + b;
                        p.nbatch = 1;
                        CK(launch_svicd(p, h->vpt, nnb, q, h->cl, grid, h->st));
                        ++launches;
                        ++klaunches;
                    }
                }
                if (int r = kev_mark(h, false)) return r;
            }
            if (h->nranks > 1 && parities == 2) {
                // slices updated in this half have global parity zp
                int r = exchange_halo(h, zp);
                if (r) return r;
            }
        }
        if (p.theta2_pass) h->theta2_ok = true;
        if (h->nranks > 1 && h->comm) {
            CKN(nccl().AllReduce(h->d_counters, h->d_counters, 4, ncclUint64, ncclSum, h->comm, h->st));
            CKN(nccl().AllReduce(h->d_sum_delta, h->d_sum_delta, 1, ncclFloat64, ncclSum, h->comm, h->st));
        }
        CK(cudaMemcpyAsync(h->h_counters, h->d_counters, 4 * sizeof(unsigned long long),
                           cudaMemcpyDeviceToHost, h->st));
        CK(cudaMemcpyAsync(h->h_counters + 4, h->d_sum_delta, sizeof(double), cudaMemcpyDeviceToHost,
                           h->st));
        CK(cudaStreamSynchronize(h->st));
        for (int i = 0; i < h->kev_used; ++i) {
            float kms = 0.f;
            CK(cudaEventElapsedTime(&kms, h->kev[2 * i], h->kev[2 * i + 1]));
            ksec += kms * 1e-3;
        }
        updates += (int64_t)h->h_counters[0];
        skipped += (int64_t)h->h_counters[1];
        visits += (int64_t)h->h_counters[2];
        empty += (int64_t)h->h_counters[3];
        double sd;
        memcpy(&sd, h->h_counters + 4, sizeof(double));
        if (!isfinite(sd)) return fail(h, MBIR_ENUMERIC, "non-finite update amount");
        sum_delta += sd;
        ++iters;
        if (n_iter < 0) {
            if (h->h_counters[2] == 0)  // nothing was scheduled: the loop could never progress
                return fail(h, MBIR_ESTATE, "an iteration scheduled no SuperVoxel (batch threshold "
                                            "drops every task: lower batch_threshold or batch_svs)");
            // no executed update: either every visited voxel was zero-skipped (a random subset
            // can be all zero while the image is not), or the image is all zero.  Stop only when
            // an iteration that visited every SV without zero-skipping executed nothing (then the
            // image is all zero and stays so), or after 16 consecutive such iterations
            zero_iters = h->h_counters[0] == 0 ? zero_iters + 1 : 0;
            const bool visited_all = (h->iter == 1 || h->o.deterministic) && !p.zero_skip_active;
            if (h->h_counters[0] == 0 && (visited_all || zero_iters >= 16)) break;
        }
    }
    CK(cudaEventRecord(h->ev1, h->st));
    CK(cudaEventSynchronize(h->ev1));
    float ms = 0.f;
    CK(cudaEventElapsedTime(&ms, h->ev0, h->ev1));
    if (st) {
        st->updates = updates;
        st->skipped = skipped;
        st->sv_visits = visits;
        st->sv_visits_empty = empty;
        st->iterations = iters;
        st->equits = (double)updates / nvox_total;
        st->seconds = ms * 1e-3;
        st->sum_abs_delta = sum_delta;
        st->launches = launches;
        st->kernel_seconds = ksec;
        st->kernel_launches = klaunches;
    }
    if (h->d_tprof) {  // development aid: per-phase cycles of the update kernel (thread 0 of each CTA)
        unsigned long long t[32];
        cudaMemcpy(t, h->d_tprof, sizeof(t), cudaMemcpyDeviceToHost);
        cudaMemset(h->d_tprof, 0, sizeof(t));
        const double v = (double)(t[5] ? t[5] : 1);
        fprintf(stderr,
                "[mbir phase] visits %llu voxels %llu | cycles/visit: order %.0f pack %.0f loop %.0f "
                "writeback %.0f | loop cycles/voxel %.1f\n",
                t[5], t[4], t[0] / v, t[1] / v, t[2] / v, t[3] / v, t[2] / (double)(t[4] ? t[4] : 1));
    }
    return MBIR_OK;
}

template <typename T>
int dalloc(mbir_handle* h, T** p, size_t n)
{
    cudaError_t e = cudaMalloc((void**)p, std::max<size_t>(n, 1) * sizeof(T));
    if (e != cudaSuccess) return fail(h, MBIR_ENOMEM, std::string("cudaMalloc: ") + cudaGetErrorString(e));
    return MBIR_OK;
}

}  // namespace

extern "C" {

void mbir_default_options(mbir_options* o)
{
    if (!o) return;
    memset(o, 0, sizeof(*o));
    o->sv_side = 9;
    o->sv_fraction = 0.25;
    o->batch_svs = 0;
    o->batch_threshold = -1;
    o->zero_skip = 1;
    o->quantize_A = 1;
    o->seed = 3000;
    o->deterministic = 0;
    o->cluster = 0;
    o->zero_skip_period = 4;
    o->voxels_per_step = 0;
}

void mbir_default_prior(mbir_prior* p)
{
    if (!p) return;
    p->p = 1.2;
    p->q = 2.0;
    p->T = 1.0;
    p->sigma = 0.005;
    p->neighborhood = 26;
    p->positivity = 1;
}

const char* mbir_strerror(int code)
{
    switch (code) {
    case MBIR_OK: return "ok";
    case MBIR_EINVAL: return "invalid argument";
    case MBIR_ENOMEM: return "out of memory";
    case MBIR_ECUDA: return "CUDA error";
    case MBIR_ESTATE: return "call out of order";
    case MBIR_ENUMERIC: return "non-finite value";
    case MBIR_ENCCL: return "NCCL error";
    case MBIR_ENOTSUP: return "not supported";
    default: return "unknown error";
    }
}

const char* mbir_last_error(const mbir_handle* h) { return h ? h->err.c_str() : "null handle"; }

int mbir_nccl_unique_id(void* id128)
{
    if (!id128) return MBIR_EINVAL;
    NcclApi& N = nccl();
    if (!N.ok) return MBIR_ENOTSUP;
    ncclUniqueId id;
    if (N.GetUniqueId(&id) != ncclSuccess) return MBIR_ENCCL;
    memcpy(id128, &id, sizeof(id));
    return MBIR_OK;
}

int mbir_halo_plan(int z_offset, int nz_local, int rank, int nranks, int parity, int32_t* ops)
{
    if (!ops || nz_local < 1 || z_offset < 0 || nranks < 1 || rank < 0 || rank >= nranks || parity < -1 ||
        parity > 1)
        return MBIR_EINVAL;
    const int z0 = z_offset, z1 = z_offset + nz_local - 1;  // my first / last global slice
    int n = 0;
    auto add = [&](int peer, int send, int slice) {
        ops[3 * n] = peer;
        ops[3 * n + 1] = send;
        ops[3 * n + 2] = slice;
        ++n;
    };
    // my first slice -> rank-1 (its upper halo), my lower halo <- rank-1's last slice (z0 - 1)
    if (rank > 0) {
        if (parity < 0 || (z0 & 1) == parity) add(rank - 1, 1, 1);
        if (parity < 0 || ((z0 - 1) & 1) == parity) add(rank - 1, 0, 0);
    }
    // my last slice -> rank+1 (its lower halo), my upper halo <- rank+1's first slice (z1 + 1)
    if (rank < nranks - 1) {
        if (parity < 0 || (z1 & 1) == parity) add(rank + 1, 1, nz_local);
        if (parity < 0 || ((z1 + 1) & 1) == parity) add(rank + 1, 0, nz_local + 1);
    }
    return n;
}

void mbir_destroy(mbir_handle* h)
{
    if (!h) return;
    if (h->st) cudaStreamSynchronize(h->st);
    void* ptrs[] = {h->A.codes, h->A.vals, h->A.off, h->A.count, h->A.scale, h->A.band_start,
                    h->A.band_width, h->d_cs, h->d_y, h->d_w, h->d_e, h->d_x, h->d_theta2,
                    h->d_scratch, h->d_amount, h->d_task_list, h->d_task_count,
                    h->d_flat, h->d_brange, h->d_fetch, h->d_gbar, h->d_keep, h->d_perm, h->d_counters, h->d_sum_delta,
                    h->d_flag, h->d_acc, h->d_tprof, h->d_dump, h->d_dump_count};
    for (void* p : ptrs)
        if (p) cudaFree(p);
    if (h->h_counters) cudaFreeHost(h->h_counters);
    if (h->ev0) cudaEventDestroy(h->ev0);
    if (h->ev1) cudaEventDestroy(h->ev1);
    for (cudaEvent_t e : h->kev) cudaEventDestroy(e);
    if (h->comm && nccl().CommDestroy) nccl().CommDestroy(h->comm);
    if (h->lg) {
        LocalGroup* g = h->lg;
        bool last = false;
        {
            std::lock_guard<std::mutex> lk(g->mu);
            g->members[h->rank] = nullptr;
            last = std::all_of(g->members.begin(), g->members.end(), [](mbir_handle* m) { return m == nullptr; });
        }
        if (last) delete g;
    }
    if (h->own_stream && h->st) cudaStreamDestroy(h->st);
    delete h;
}

int mbir_create(const mbir_geometry* g, const mbir_prior* pr, const mbir_options* o,
                const mbir_dist* d, mbir_handle** out)
{
    if (!out) return MBIR_EINVAL;
    *out = nullptr;
    if (!g) return MBIR_EINVAL;
    mbir_handle* h = new (std::nothrow) mbir_handle();
    if (!h) return MBIR_ENOMEM;
    auto bail = [&](int code) {
        mbir_destroy(h);
        return code;
    };
    h->g = *g;
    if (pr)
        h->pr = *pr;
    else
        mbir_default_prior(&h->pr);
    if (o)
        h->o = *o;
    else
        mbir_default_options(&h->o);
    if (d) {
        h->device = d->device;
        h->st = (cudaStream_t)d->stream;
        h->rank = d->rank;
        h->nranks = d->nranks < 1 ? 1 : d->nranks;
    }
    // ---- validation (MBIR_EINVAL)
    const mbir_geometry& G = h->g;
    if (G.nz_total <= 0) h->g.nz_total = G.nz_local;
    if (G.nx < 1 || G.ny < 1 || G.nz_local < 1 || G.nviews < 1 || G.nchannels < 1 || !(G.dxy > 0) ||
        !(G.dchannel > 0) || G.z_offset < 0 || G.z_offset + G.nz_local > h->g.nz_total)
        return bail(MBIR_EINVAL);
    if (G.nviews > 768) return (fail(h, MBIR_EINVAL, "nviews > 768 not supported"), bail(MBIR_EINVAL));
    if (G.nchannels > (1 << 24)) return bail(MBIR_EINVAL);
    const mbir_prior& P = h->pr;
    if (!(P.p >= 1.0 && P.p <= 2.0) || P.q != 2.0 || !(P.T > 0) || !(P.sigma > 0) ||
        (P.neighborhood != 8 && P.neighborhood != 26))
        return bail(MBIR_EINVAL);
    if (h->o.sv_side < 1 || h->o.sv_side > 16 || !(h->o.sv_fraction > 0 && h->o.sv_fraction <= 1) ||
        h->o.batch_svs < 0 || h->o.zero_skip_period < 0)
        return bail(MBIR_EINVAL);
    {
        // the phase task lists (sched.cu k_flatten) gather at most kMaxPhaseSlices slices of one
        // z-parity: reject larger slabs instead of leaving slices unscheduled
        const int parities = (P.neighborhood == 26 && h->g.nz_total > 1) ? 2 : 1;
        if ((G.nz_local + parities - 1) / parities > kMaxPhaseSlices)
            return (fail(h, MBIR_EINVAL, "nz_local too large: at most " + std::to_string(kMaxPhaseSlices) +
                                             " slices per z-parity phase per rank"), bail(MBIR_EINVAL));
    }
    // nranks > 1 needs an NCCL id -- or none, for slabs linked on one device by mbir_link_slabs
    if (h->nranks > 1 && (!d || h->rank < 0 || h->rank >= h->nranks))
        return bail(MBIR_EINVAL);
    if (G.angles) h->angles.assign(G.angles, G.angles + G.nviews);
    h->g.angles = nullptr;

    if (cudaSetDevice(h->device) != cudaSuccess) return bail(MBIR_ECUDA);
    if (!h->st) {
        // a BLOCKING stream: its work is ordered after (and before) work on the legacy default
        // stream, so device inputs produced there (e.g. torch tensors on torch's default stream)
        // are complete before the library reads them
        if (cudaStreamCreateWithFlags(&h->st, cudaStreamDefault) != cudaSuccess) return bail(MBIR_ECUDA);
        h->own_stream = true;
    }
    int r;
    cudaDeviceProp prop;
    if (cudaGetDeviceProperties(&prop, h->device) != cudaSuccess) return bail(MBIR_ECUDA);
    h->nsm = prop.multiProcessorCount;

    // ---- SuperVoxel tiling (reading R13: ceil tiles, no overlap)
    h->side = h->o.sv_side;
    h->S2 = h->side * h->side;
    h->nsvx = (G.nx + h->side - 1) / h->side;
    h->nsvy = (G.ny + h->side - 1) / h->side;
    h->nsv = h->nsvx * h->nsvy;
    if (h->nsv > 16384) return (fail(h, MBIR_EINVAL, "too many SuperVoxels per slice (> 16384)"), bail(MBIR_EINVAL));
    h->nsv_pad = 1;
    while (h->nsv_pad < h->nsv) h->nsv_pad <<= 1;
    h->max_group = ((h->nsvx + 1) / 2) * ((h->nsvy + 1) / 2);

    // ---- view angles as (cos, sin) in double, computed on the host
    {
        std::vector<double> cs(2 * (size_t)G.nviews);
        for (int k = 0; k < G.nviews; ++k) {
            const double th = h->angles.empty() ? (double)k * 3.14159265358979323846 / (double)G.nviews : h->angles[k];
            cs[2 * k] = cos(th);
            cs[2 * k + 1] = sin(th);
        }
        if ((r = dalloc(h, &h->d_cs, cs.size()))) return bail(r);
        if (cudaMemcpy(h->d_cs, cs.data(), cs.size() * 8, cudaMemcpyHostToDevice) != cudaSuccess) return bail(MBIR_ECUDA);
    }

    // ---- system matrix, compressed per SV (a1)
    const bool quant = h->o.quantize_A != 0;
    h->A.nsv = h->nsv;
    h->A.S2 = h->S2;
    h->A.V = G.nviews;
    // ---- update-kernel shape: fat view warps (4 views per lane, <= 6 warps) keep the per-voxel
    // per-warp overhead (reduction, barrier, delta) small; <= 128 views use 1 view per lane
    // (<= 4 warps)
    h->vpt = G.nviews > 128 ? MBIR_WIDE_VPT : 1;
    h->nvw = (G.nviews + 32 * h->vpt - 1) / (32 * h->vpt);
    if (h->nvw * h->vpt > 24) return (fail(h, MBIR_EINVAL, "nviews > 768 not supported"), bail(MBIR_EINVAL));
    // an explicit 2-CTA cluster splits the view warps evenly: an odd count is padded by one warp
    // whose views (>= nviews) carry zero records (no loads, no contribution)
    if (h->vpt == MBIR_WIDE_VPT && (h->nvw & 1) && h->o.cluster == 2) h->nvw += 1;
    size_t nA = 0;
    for (int attempt = 0;; ++attempt) {
    h->Vs = (h->nvw * 32 * h->vpt + 127) / 128 * 128;  // record stride: whole 128-view tiles
    h->A.vpt = h->vpt;
    h->A.VA = h->Vs;  // thread-major record positions (apos); a multiple of 32 -> TMA-sized
    nA = (size_t)h->nsv * h->S2 * h->A.VA;
    if (quant) {
        if ((r = dalloc(h, &h->A.codes, nA))) return bail(r);
        cudaMemsetAsync(h->A.codes, 0, nA * 4, h->st);
    } else {
        if ((r = dalloc(h, &h->A.vals, nA))) return bail(r);
        cudaMemsetAsync(h->A.vals, 0, nA * 16, h->st);
    }
    if ((r = dalloc(h, &h->A.off, nA))) return bail(r);
    if ((r = dalloc(h, &h->A.count, nA))) return bail(r);
    cudaMemsetAsync(h->A.off, 0, nA, h->st);
    cudaMemsetAsync(h->A.count, 0, nA, h->st);
    if ((r = dalloc(h, &h->A.scale, (size_t)h->nsv * h->S2))) return bail(r);
    if ((r = dalloc(h, &h->A.band_start, (size_t)h->nsv * G.nviews))) return bail(r);
    if ((r = dalloc(h, &h->A.band_width, (size_t)h->nsv * G.nviews))) return bail(r);
    int* d_info = nullptr;  // [err, maxrow, maxwidth]
    if ((r = dalloc(h, &d_info, 3))) return bail(r);
    cudaMemsetAsync(d_info, 0, 3 * sizeof(int), h->st);
    if (build_sysmatrix(h->g, h->d_cs, h->side, h->nsvx, h->nsvy, quant, h->A, d_info, d_info + 1, h->st) != cudaSuccess) {
        cudaFree(d_info);
        return (fail(h, MBIR_ECUDA, "system matrix build failed"), bail(MBIR_ECUDA));
    }
    int info[3] = {0, 0, 0};
    cudaMemcpyAsync(info, d_info, sizeof(info), cudaMemcpyDeviceToHost, h->st);
    if (cudaStreamSynchronize(h->st) != cudaSuccess) {
        cudaFree(d_info);
        return bail(MBIR_ECUDA);
    }
    cudaFree(d_info);
    if (info[0] & 1) return (fail(h, MBIR_EINVAL, "a voxel meets more than 4 channels in one view (dchannel too small vs dxy)"), bail(MBIR_EINVAL));
    if (info[0] & 2) return (fail(h, MBIR_EINVAL, "SV band wider than 255 channels"), bail(MBIR_EINVAL));
    h->rows = info[1];
    h->band_max = info[2];
    // a band row plus its misalignment (<= 3 floats) must fit one or two aligned 32-float windows
    if (h->rows > kMaxSvbRows - 3)
        return (fail(h, MBIR_EINVAL, "SV band needs " + std::to_string(h->rows) + " > 61 buffer rows: reduce sv_side"), bail(MBIR_EINVAL));
    h->nwin = h->rows + 3 > 32 ? 2 : 1;
    // automatic cluster (below) for a buffer one CTA cannot hold, with an odd view-warp count:
    // rebuild A once with the count padded to even
    if (attempt == 0 && h->o.cluster == 0 && h->vpt == MBIR_WIDE_VPT && (h->nvw & 1)) {
        IcdParams t = make_params(h);
        t.A.VA = h->Vs;
        if (svicd_smem_bytes(t, h->vpt, P.neighborhood, quant, 1) > (int)prop.sharedMemPerBlockOptin) {
            void* ptrs[] = {h->A.codes, h->A.vals, h->A.off, h->A.count, h->A.scale, h->A.band_start, h->A.band_width};
            for (void* q : ptrs)
                if (q) cudaFree(q);
            h->A.codes = nullptr;
            h->A.vals = nullptr;
            h->A.off = h->A.count = nullptr;
            h->A.scale = nullptr;
            h->A.band_start = nullptr;
            h->A.band_width = nullptr;
            h->nvw += 1;
            continue;
        }
    }
    break;
    }
    h->a_bytes = (int64_t)nA * ((quant ? 4 : 16) + 2) + (int64_t)h->nsv * h->S2 * 4 + (int64_t)h->nsv * G.nviews * 5;

    {
        // the fused update kernel: nvw view warps + the delta warp + the prior warp per task; the
        // task's CTA owns all views (cluster 1) or a 2-CTA cluster splits them (cluster 2: each
        // CTA holds half the views' SV buffer and exchanges one partial sum per voxel through
        // distributed shared memory -- two SMs per SV for few-SV (2-D) workloads)
        IcdParams p = make_params(h);
        if (h->o.cluster < 0 || h->o.cluster > 2)
            return (fail(h, MBIR_EINVAL, "cluster must be 0 (auto), 1 or 2"), bail(MBIR_EINVAL));
        h->cl = h->o.cluster == 2 ? 2 : 1;
        // auto: a 2-CTA cluster when one CTA cannot hold the SV buffer (large SVs, NEXT-2)
        if (h->o.cluster == 0 && h->vpt == MBIR_WIDE_VPT && h->nvw % 2 == 0 &&
            svicd_smem_bytes(p, h->vpt, P.neighborhood, quant, 1) > (int)prop.sharedMemPerBlockOptin)
            h->cl = 2;
        if (h->cl == 2 && !(h->vpt == 4 && h->nvw % 2 == 0))
            return (fail(h, MBIR_EINVAL, "cluster = 2 needs > 128 views in an even number of 128-view warps"), bail(MBIR_EINVAL));
        if (h->o.voxels_per_step < 0 || h->o.voxels_per_step > 2)
            return (fail(h, MBIR_EINVAL, "voxels_per_step must be 0 (auto), 1 or 2"), bail(MBIR_EINVAL));
        if (h->o.voxels_per_step == 2 && (h->cl == 2 || !quant))
            return (fail(h, MBIR_EINVAL, "voxels_per_step = 2 needs uint8 A (quantize_A) and one CTA per task"), bail(MBIR_EINVAL));
        h->kv = h->o.voxels_per_step ? h->o.voxels_per_step : 1;  // auto: exact steps (pairs measured slower)
        h->threads = 32 * (h->nvw / h->cl + 2);
        h->smem = svicd_smem_bytes(p, h->vpt, P.neighborhood, quant, h->cl);
        if (h->smem > (int)prop.sharedMemPerBlockOptin)
            return (fail(h, MBIR_EINVAL, "SV buffer (" + std::to_string(h->smem) + " B) exceeds shared memory: reduce sv_side"), bail(MBIR_EINVAL));
        h->resident = svicd_resident_ctas(p, h->vpt, P.neighborhood, quant, h->cl);
        if (h->resident <= 0) return (fail(h, MBIR_ECUDA, "update kernel does not fit on the device"), bail(MBIR_ECUDA));
        h->blocks_per_sm = std::max(1, (h->resident + h->nsm - 1) / h->nsm);
    }

    // ---- state buffers
    const size_t ns = sino_elems(h), pl = plane_elems(h);
    // (+64 floats: the update kernel reads whole 32-float windows around band rows, up to 64
    // floats past the last row with two windows; the padding is zero, never uninitialised)
    if ((r = dalloc(h, &h->d_y, ns + 64))) return bail(r);
    if ((r = dalloc(h, &h->d_w, ns + 64))) return bail(r);
    if ((r = dalloc(h, &h->d_e, ns + 64))) return bail(r);
    cudaMemsetAsync(h->d_y, 0, (ns + 64) * 4, h->st);
    cudaMemsetAsync(h->d_w, 0, (ns + 64) * 4, h->st);
    cudaMemsetAsync(h->d_e, 0, (ns + 64) * 4, h->st);
    if ((r = dalloc(h, &h->d_x, pl * (G.nz_local + 2)))) return bail(r);
    if ((r = dalloc(h, &h->d_theta2, (size_t)G.nz_local * h->nsv * h->S2))) return bail(r);
    cudaMemset(h->d_theta2, 0, (size_t)G.nz_local * h->nsv * h->S2 * sizeof(float));
    if ((r = dalloc(h, &h->d_amount, (size_t)G.nz_local * h->nsv))) return bail(r);
    // e_init tiles of the concurrently running SV visits: one per CTA of the largest grid
    if ((r = dalloc(h, &h->d_scratch, (size_t)h->nsm * h->blocks_per_sm * svicd_scratch_floats(h->vpt, h->nwin)))) return bail(r);
    if ((r = dalloc(h, &h->d_task_list, (size_t)G.nz_local * 4 * h->max_group))) return bail(r);
    if ((r = dalloc(h, &h->d_task_count, (size_t)G.nz_local * 4))) return bail(r);
    if ((r = dalloc(h, &h->d_flat, (size_t)8 * G.nz_local * h->max_group))) return bail(r);
    if ((r = dalloc(h, &h->d_brange, (size_t)8 * (h->max_group + 1)))) return bail(r);
    if ((r = dalloc(h, &h->d_keep, (size_t)G.nz_local * h->max_group))) return bail(r);
    if ((r = dalloc(h, &h->d_fetch, (size_t)8 * h->max_group))) return bail(r);
    if ((r = dalloc(h, &h->d_gbar, 8))) return bail(r);
    {
        // random voxel visiting orders within an SV ("randomized order"; reading R10):
        // kNPerm Fisher-Yates permutations from a seeded splitmix64, one picked per SV visit
        std::vector<uint8_t> perm((size_t)mbir_handle::kNPerm * h->S2);
        uint64_t s = h->o.seed ^ 0xA0761D6478BD642FULL;
        auto next = [&s]() {
            uint64_t z = (s += 0x9E3779B97F4A7C15ULL);
            z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
            z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
            return z ^ (z >> 31);
        };
        for (int q = 0; q < mbir_handle::kNPerm; ++q) {
            uint8_t* pq = perm.data() + (size_t)q * h->S2;
            for (int i = 0; i < h->S2; ++i) pq[i] = (uint8_t)i;
            for (int i = h->S2 - 1; i > 0; --i) std::swap(pq[i], pq[next() % (uint64_t)(i + 1)]);
        }
        if ((r = dalloc(h, &h->d_perm, perm.size()))) return bail(r);
        if (cudaMemcpy(h->d_perm, perm.data(), perm.size(), cudaMemcpyHostToDevice) != cudaSuccess) return bail(MBIR_ECUDA);
    }
    if ((r = dalloc(h, &h->d_counters, 4))) return bail(r);
    if ((r = dalloc(h, &h->d_sum_delta, 1))) return bail(r);
    if ((r = dalloc(h, &h->d_flag, 1))) return bail(r);
    if ((r = dalloc(h, &h->d_acc, 1))) return bail(r);
    if (getenv("MBIR_PHASE_PROFILE")) {
        if ((r = dalloc(h, &h->d_tprof, 32))) return bail(r);
        cudaMemset(h->d_tprof, 0, 32 * sizeof(unsigned long long));
    }
    if (cudaMallocHost((void**)&h->h_counters, 5 * sizeof(unsigned long long)) != cudaSuccess) return bail(MBIR_ENOMEM);
    cudaMemsetAsync(h->d_x, 0, sizeof(float) * pl * (G.nz_local + 2), h->st);
    cudaMemsetAsync(h->d_amount, 0, sizeof(float) * G.nz_local * h->nsv, h->st);
    if (cudaEventCreate(&h->ev0) != cudaSuccess || cudaEventCreate(&h->ev1) != cudaSuccess) return bail(MBIR_ECUDA);

    // ---- prior constants (reading R1-R2)
    {
        PriorConst pc{};
        int n = 0;
        for (int dz = -1; dz <= 1; ++dz)
            for (int dy = -1; dy <= 1; ++dy)
                for (int dx = -1; dx <= 1; ++dx) {
                    if (dx == 0 && dy == 0 && dz == 0) continue;
                    if (P.neighborhood == 8 && dz != 0) continue;
                    const int m = abs(dx) + abs(dy) + abs(dz);
                    const double norm = P.neighborhood == 8 ? 4.0 + 4.0 / sqrt(2.0)
                                                            : 6.0 + 12.0 / sqrt(2.0) + 8.0 / sqrt(3.0);
                    pc.dx[n] = dx;
                    pc.dy[n] = dy;
                    pc.dz[n] = dz;
                    pc.b[n] = (float)((1.0 / sqrt((double)m)) / norm);
                    ++n;
                }
        pc.nnb = n;
        pc.c_phi = (float)(1.0 / (2.0 * pow(P.sigma, P.p) * pow(P.T * P.sigma, P.q - P.p)));
        pc.pq = (float)(P.q / P.p);
        pc.qmp = (float)(P.q - P.p);
        pc.inv_Ts = (float)(1.0 / (P.T * P.sigma));
        pc.positivity = P.positivity;
        h->pc = pc;
    }

    // ---- multi-GPU communicator (z-slab partition)
    if (h->nranks > 1 && d->nccl_unique_id) {
        NcclApi& N = nccl();
        if (!N.ok) return (fail(h, MBIR_ENOTSUP, "libnccl.so.2 not found"), bail(MBIR_ENOTSUP));
        ncclUniqueId id;
        memcpy(&id, d->nccl_unique_id, sizeof(id));
        if (N.CommInitRank(&h->comm, h->nranks, id, h->rank) != ncclSuccess)
            return (fail(h, MBIR_ENCCL, "ncclCommInitRank failed"), bail(MBIR_ENCCL));
    }
    if (cudaStreamSynchronize(h->st) != cudaSuccess) return bail(MBIR_ECUDA);
    {
        // nnz and band statistics (for the roofline accounting)
        std::vector<uint8_t> cnt(nA), bw((size_t)h->nsv * G.nviews);
        cudaMemcpy(cnt.data(), h->A.count, nA, cudaMemcpyDeviceToHost);
        cudaMemcpy(bw.data(), h->A.band_width, bw.size(), cudaMemcpyDeviceToHost);
        int64_t s = 0, b = 0;
        for (uint8_t c : cnt) s += c;
        for (uint8_t c : bw) b += c;
        h->nnz = s;
        h->band_entries = b;
    }
    *out = h;
    return MBIR_OK;
}

int mbir_set_sinogram(mbir_handle* h, const float* y, const float* w, int where)
{
    if (!h || !y || !w) return MBIR_EINVAL;
    const size_t ns = sino_elems(h);
    CK(cudaMemcpyAsync(h->d_y, y, ns * 4, kind_in(where), h->st));
    CK(cudaMemcpyAsync(h->d_w, w, ns * 4, kind_in(where), h->st));
    CK(cudaMemsetAsync(h->d_flag, 0, sizeof(int), h->st));
    CK(launch_check_finite(h->d_y, (int64_t)ns, 0, h->d_flag, h->st));
    CK(launch_check_finite(h->d_w, (int64_t)ns, 1, h->d_flag, h->st));
    int flag = 0;
    CK(cudaMemcpyAsync(&flag, h->d_flag, sizeof(int), cudaMemcpyDeviceToHost, h->st));
    CK(cudaStreamSynchronize(h->st));
    if (flag) {
        h->have_sino = false;
        return fail(h, MBIR_EINVAL, "y must be finite and w finite and >= 0");
    }
    int r = refresh_error(h);  // theta2 follows in the first iteration (run_iterations)
    if (r) return r;
    h->theta2_ok = false;
    CK(cudaMemsetAsync(h->d_amount, 0, sizeof(float) * h->g.nz_local * h->nsv, h->st));
    CK(cudaStreamSynchronize(h->st));
    h->have_sino = true;
    h->iter = 0;
    return MBIR_OK;
}

int mbir_set_image(mbir_handle* h, const float* x0, int where)
{
    if (!h) return MBIR_EINVAL;
    const size_t pl = plane_elems(h);
    if (x0) {
        // validate in a temporary buffer first: on rejection the image, e and the scheduler
        // state stay untouched (e = y - A x keeps holding).  The verdict is agreed across ranks
        // before anyone returns, so a rejecting rank cannot leave the others in the collective
        // halo exchange below.
        const size_t n = pl * h->g.nz_local;
        float* tmp = nullptr;
        CK(cudaMallocAsync((void**)&tmp, n * 4, h->st));
        CK(cudaMemcpyAsync(tmp, x0, n * 4, kind_in(where), h->st));
        CK(cudaMemsetAsync(h->d_flag, 0, sizeof(int), h->st));
        CK(launch_check_finite(tmp, (int64_t)n, h->pr.positivity, h->d_flag, h->st));
        if (h->comm) CKN(nccl().AllReduce(h->d_flag, h->d_flag, 1, ncclInt32, ncclMax, h->comm, h->st));
        int flag = 0;
        CK(cudaMemcpyAsync(&flag, h->d_flag, sizeof(int), cudaMemcpyDeviceToHost, h->st));
        CK(cudaStreamSynchronize(h->st));
        if (!flag) CK(cudaMemcpyAsync(h->d_x + pl, tmp, n * 4, cudaMemcpyDeviceToDevice, h->st));
        CK(cudaFreeAsync(tmp, h->st));
        if (flag) {
            CK(cudaStreamSynchronize(h->st));
            return fail(h, MBIR_EINVAL, "x0 must be finite (and >= 0 with positivity) on every rank");
        }
    } else {
        CK(cudaMemsetAsync(h->d_x + pl, 0, pl * h->g.nz_local * 4, h->st));
    }
    h->x_zero = (x0 == nullptr);
    int r = exchange_halo(h, -1);
    if (r) return r;
    if (h->have_sino) {
        r = refresh_error(h);
        if (r) return r;
    }
    CK(cudaMemsetAsync(h->d_amount, 0, sizeof(float) * h->g.nz_local * h->nsv, h->st));
    CK(cudaStreamSynchronize(h->st));
    h->iter = 0;
    return MBIR_OK;
}

int mbir_init_fbp(mbir_handle* h)
{
    if (!h) return MBIR_EINVAL;
    if (!h->have_sino) return fail(h, MBIR_ESTATE, "mbir_set_sinogram has not been called");
    const size_t pl = plane_elems(h);
    // the filtered sinogram lives in e, which is recomputed (e = y - A x) right after: no
    // allocation per call (a stream-ordered malloc/free of the sinogram size cost up to 50 ms)
    cudaError_t e = launch_fbp(h->g, h->d_cs, h->d_y, h->d_e, h->d_x + pl, h->pr.positivity, h->st);
    if (e != cudaSuccess) return fail(h, MBIR_ECUDA, std::string("FBP: ") + cudaGetErrorString(e));
    h->x_zero = false;
    int r = exchange_halo(h, -1);
    if (r) return r;
    r = refresh_error(h);
    if (r) return r;
    CK(cudaMemsetAsync(h->d_amount, 0, sizeof(float) * h->g.nz_local * h->nsv, h->st));
    CK(cudaStreamSynchronize(h->st));
    h->iter = 0;
    return MBIR_OK;
}

int mbir_reconstruct(mbir_handle* h, double equits, mbir_stats* st)
{
    if (!h || !(equits >= 0)) return MBIR_EINVAL;
    // linked slabs do not reduce their counters, so an equit target could stop them after
    // different iteration counts: they run fixed iteration counts (mbir_iterate)
    if (h->lg) return fail(h, MBIR_ENOTSUP, "linked slabs (mbir_link_slabs) run mbir_iterate only");
    return run_iterations(h, -1, equits, st);
}

int mbir_iterate(mbir_handle* h, int n_iterations, mbir_stats* st)
{
    if (!h || n_iterations < 0) return MBIR_EINVAL;
    return run_iterations(h, n_iterations, 0.0, st);
}

int mbir_get_image(mbir_handle* h, float* x, int where)
{
    if (!h || !x) return MBIR_EINVAL;
    const size_t pl = plane_elems(h);
    CK(cudaMemcpyAsync(x, h->d_x + pl, pl * h->g.nz_local * 4, kind_out(where), h->st));
    CK(cudaStreamSynchronize(h->st));
    return MBIR_OK;
}

int mbir_get_error_sinogram(mbir_handle* h, float* e, int where)
{
    if (!h || !e) return MBIR_EINVAL;
    CK(cudaMemcpyAsync(e, h->d_e, sino_elems(h) * 4, kind_out(where), h->st));
    CK(cudaStreamSynchronize(h->st));
    return MBIR_OK;
}

int mbir_rmse_hu(mbir_handle* h, const float* golden, int where, double mu_water, double* out)
{
    if (!h || !golden || !out || !(mu_water > 0)) return MBIR_EINVAL;
    const size_t pl = plane_elems(h), n = pl * h->g.nz_local;
    const float* g = golden;
    float* tmp = nullptr;
    if (where != MBIR_DEVICE) {
        CK(cudaMallocAsync((void**)&tmp, n * 4, h->st));
        CK(cudaMemcpyAsync(tmp, golden, n * 4, cudaMemcpyHostToDevice, h->st));
        g = tmp;
    }
    CK(cudaMemsetAsync(h->d_acc, 0, sizeof(double), h->st));
    CK(launch_rmse_partial(h->d_x + pl, g, (int64_t)n, h->d_acc, h->st));
    if (h->comm) CKN(nccl().AllReduce(h->d_acc, h->d_acc, 1, ncclFloat64, ncclSum, h->comm, h->st));
    double s = 0.0;
    CK(cudaMemcpyAsync(&s, h->d_acc, sizeof(double), cudaMemcpyDeviceToHost, h->st));
    if (tmp) CK(cudaFreeAsync(tmp, h->st));
    CK(cudaStreamSynchronize(h->st));
    *out = 1000.0 * sqrt(s / ((double)pl * h->g.nz_total)) / mu_water;
    return MBIR_OK;
}

int mbir_query_sizes(const mbir_handle* h, mbir_sizes* s)
{
    if (!h || !s) return MBIR_EINVAL;
    s->nsv_x = h->nsvx;
    s->nsv_y = h->nsvy;
    s->nsv = h->nsv;
    s->K = kK;
    s->band_max = h->band_max;
    s->svb_rows = h->rows;
    s->threads_per_cta = h->threads;
    s->cluster = h->cl;
    s->resident_ctas = h->resident;
    s->smem_bytes = h->smem;
    s->nnz = h->nnz;
    s->a_bytes = h->a_bytes;
    s->band_entries = h->band_entries;
    s->max_group = h->max_group;
    s->voxels_per_step = h->kv;
    return MBIR_OK;
}

static int export_sysmatrix(mbir_handle* h, const int64_t* voxels, int nvox, int32_t* first,
                            int32_t* count, float* values, uint8_t* codes, float* scales)
{
    const size_t n = voxels ? (size_t)nvox : plane_elems(h), V = h->g.nviews;
    int32_t *df = nullptr, *dc = nullptr;
    float *dv = nullptr, *ds = nullptr;
    uint8_t* dq = nullptr;
    int64_t* dvox = nullptr;
    int rc = MBIR_OK;
    auto cleanup = [&]() {
        if (df) cudaFree(df);
        if (dc) cudaFree(dc);
        if (dv) cudaFree(dv);
        if (ds) cudaFree(ds);
        if (dq) cudaFree(dq);
        if (dvox) cudaFree(dvox);
    };
    if ((first && (rc = dalloc(h, &df, n * V))) || (count && (rc = dalloc(h, &dc, n * V))) ||
        (values && (rc = dalloc(h, &dv, n * V * kK))) || (codes && (rc = dalloc(h, &dq, n * V * kK))) ||
        (scales && (rc = dalloc(h, &ds, n))) || (voxels && (rc = dalloc(h, &dvox, n)))) {
        cleanup();
        return rc;
    }
    cudaError_t e = cudaSuccess;
    if (voxels) e = cudaMemcpyAsync(dvox, voxels, n * 8, cudaMemcpyHostToDevice, h->st);
    if (e == cudaSuccess)
        e = launch_export_sysmatrix(h->A, h->g.nx, h->g.ny, h->side, h->nsvx, dvox, (int)n, df, dc, dv,
                                    dq, ds, h->g, h->d_cs, h->st);
    if (e == cudaSuccess && first) e = cudaMemcpyAsync(first, df, n * V * 4, cudaMemcpyDeviceToHost, h->st);
    if (e == cudaSuccess && count) e = cudaMemcpyAsync(count, dc, n * V * 4, cudaMemcpyDeviceToHost, h->st);
    if (e == cudaSuccess && values) e = cudaMemcpyAsync(values, dv, n * V * kK * 4, cudaMemcpyDeviceToHost, h->st);
    if (e == cudaSuccess && codes) e = cudaMemcpyAsync(codes, dq, n * V * kK, cudaMemcpyDeviceToHost, h->st);
    if (e == cudaSuccess && scales) e = cudaMemcpyAsync(scales, ds, n * 4, cudaMemcpyDeviceToHost, h->st);
    if (e == cudaSuccess) e = cudaStreamSynchronize(h->st);
    cleanup();
    if (e != cudaSuccess) return fail(h, MBIR_ECUDA, cudaGetErrorString(e));
    return MBIR_OK;
}

int mbir_get_sysmatrix(mbir_handle* h, int32_t* first, int32_t* count, float* values,
                       uint8_t* codes, float* scales)
{
    if (!h) return MBIR_EINVAL;
    return export_sysmatrix(h, nullptr, 0, first, count, values, codes, scales);
}

int mbir_get_sysmatrix_columns(mbir_handle* h, const int64_t* voxels, int n, int32_t* first,
                               int32_t* count, float* values, uint8_t* codes, float* scales)
{
    if (!h || !voxels || n <= 0) return MBIR_EINVAL;
    for (int i = 0; i < n; ++i)
        if (voxels[i] < 0 || voxels[i] >= (int64_t)plane_elems(h)) return fail(h, MBIR_EINVAL, "voxel index out of range");
    return export_sysmatrix(h, voxels, n, first, count, values, codes, scales);
}

int mbir_link_slabs(mbir_handle** hs, int n)
{
    if (!hs || n < 2) return MBIR_EINVAL;
    for (int i = 0; i < n; ++i) {
        mbir_handle* h = hs[i];
        if (!h || h->nranks != n || h->rank != i || h->comm || h->lg) return MBIR_EINVAL;
        if (h->device != hs[0]->device) return fail(h, MBIR_EINVAL, "linked slabs must share one device");
        if (i > 0 && h->g.z_offset != hs[i - 1]->g.z_offset + hs[i - 1]->g.nz_local)
            return fail(h, MBIR_EINVAL, "linked slabs must be consecutive in rank order");
    }
    LocalGroup* g = new (std::nothrow) LocalGroup();
    if (!g) return MBIR_ENOMEM;
    g->n = n;
    g->members.assign(hs, hs + n);
    for (int i = 0; i < n; ++i) hs[i]->lg = g;
    return MBIR_OK;
}

int mbir_set_update_dump(mbir_handle* h, int64_t capacity)
{
    if (!h || capacity < 0) return MBIR_EINVAL;
    CK(cudaStreamSynchronize(h->st));
    if (h->d_dump) cudaFree(h->d_dump);
    if (h->d_dump_count) cudaFree(h->d_dump_count);
    h->d_dump = nullptr;
    h->d_dump_count = nullptr;
    h->dump_cap = 0;
    if (capacity == 0) return MBIR_OK;
    int r;
    if ((r = dalloc(h, &h->d_dump, (size_t)capacity * 4))) return r;
    if ((r = dalloc(h, &h->d_dump_count, 1))) return r;
    CK(cudaMemsetAsync(h->d_dump_count, 0, sizeof(unsigned long long), h->st));
    CK(cudaStreamSynchronize(h->st));
    h->dump_cap = capacity;
    return MBIR_OK;
}

int mbir_get_update_dump(mbir_handle* h, int64_t cap, int64_t* voxels, float* theta1, float* theta2,
                         float* delta, int64_t* n)
{
    if (!h || cap < 0 || !n || (cap > 0 && (!voxels || !theta1 || !theta2 || !delta))) return MBIR_EINVAL;
    if (!h->d_dump) return fail(h, MBIR_ESTATE, "mbir_set_update_dump has not been called");
    unsigned long long cnt = 0;
    CK(cudaMemcpyAsync(&cnt, h->d_dump_count, sizeof(cnt), cudaMemcpyDeviceToHost, h->st));
    CK(cudaStreamSynchronize(h->st));
    const int64_t m = std::min<int64_t>({(int64_t)cnt, cap, h->dump_cap});
    std::vector<float> buf((size_t)m * 4);
    if (m > 0) CK(cudaMemcpy(buf.data(), h->d_dump, (size_t)m * 16, cudaMemcpyDeviceToHost));
    for (int64_t i = 0; i < m; ++i) {
        uint32_t v;
        memcpy(&v, &buf[4 * i], 4);
        // bit 31: the update was computed from the same state as the record before it (pairs)
        voxels[i] = (int64_t)(v & 0x7fffffffu) | ((v >> 31) ? MBIR_DUMP_SAME_STATE : 0);
        theta1[i] = buf[4 * i + 1];
        theta2[i] = buf[4 * i + 2];
        delta[i] = buf[4 * i + 3];
    }
    *n = (int64_t)cnt;
    CK(cudaMemsetAsync(h->d_dump_count, 0, sizeof(unsigned long long), h->st));
    CK(cudaStreamSynchronize(h->st));
    return MBIR_OK;
}

int mbir_get_schedule(mbir_handle* h, int32_t* task_list, int32_t* task_count, float* amount)
{
    if (!h) return MBIR_EINVAL;
    const size_t nz = h->g.nz_local;
    if (task_list)
        CK(cudaMemcpyAsync(task_list, h->d_task_list, nz * 4 * h->max_group * 4, cudaMemcpyDeviceToHost, h->st));
    if (task_count) CK(cudaMemcpyAsync(task_count, h->d_task_count, nz * 4 * 4, cudaMemcpyDeviceToHost, h->st));
    if (amount) CK(cudaMemcpyAsync(amount, h->d_amount, nz * h->nsv * 4, cudaMemcpyDeviceToHost, h->st));
    CK(cudaStreamSynchronize(h->st));
    return MBIR_OK;
}

int mbir_probe_update(mbir_handle* h, const int64_t* voxels, int n, float* theta1, float* theta2,
                      float* delta)
{
    if (!h || !voxels || n <= 0 || !theta1 || !theta2 || !delta) return MBIR_EINVAL;
    if (!h->have_sino) return fail(h, MBIR_ESTATE, "mbir_set_sinogram has not been called");
    const int64_t nv = (int64_t)plane_elems(h) * h->g.nz_local;
    for (int i = 0; i < n; ++i)
        if (voxels[i] < 0 || voxels[i] >= nv) return fail(h, MBIR_EINVAL, "voxel index out of range");
    int64_t* dvox = nullptr;
    float* dout = nullptr;
    CK(cudaMallocAsync((void**)&dvox, n * 8, h->st));
    CK(cudaMallocAsync((void**)&dout, n * 12, h->st));
    CK(cudaMemcpyAsync(dvox, voxels, n * 8, cudaMemcpyHostToDevice, h->st));
    IcdParams p = make_params(h);
    CK(launch_probe(p, h->o.quantize_A != 0, h->pr.neighborhood, dvox, n, dout, h->st));
    std::vector<float> out((size_t)n * 3);
    CK(cudaMemcpyAsync(out.data(), dout, n * 12, cudaMemcpyDeviceToHost, h->st));
    CK(cudaFreeAsync(dvox, h->st));
    CK(cudaFreeAsync(dout, h->st));
    CK(cudaStreamSynchronize(h->st));
    for (int i = 0; i < n; ++i) {
        theta1[i] = out[3 * i];
        theta2[i] = out[3 * i + 1];
        delta[i] = out[3 * i + 2];
    }
    return MBIR_OK;
}

}  // extern "C"
