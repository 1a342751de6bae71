#!/usr/bin/env python
"""Benchmark of the GPU-ICD hot path (BASELINE.json metric: voxel updates/s and
time-to-converge (< 10 HU RMSE) per volume at 1/2/4/8 B200).

Workload (BASELINE.json configs[3], fits one GPU): 512 x 512 x 64 volume, 720 views x 1024
channels parallel beam, 3-D Shepp-Logan with Poisson noise (lambda0 = 1e4), q-GGMRF prior over
the 26-neighbourhood, SuperVoxel side 9, uint8 A.  N GPUs: z-slabs of 64/N slices with the
NCCL halo exchange (strong scaling of one fixed volume).

A "step" = one reconstruction from x0 = 0 of E equits (set_image(0) + mbir_reconstruct(E));
value = executed voxel updates (all ranks) / max-over-ranks device time of K steps.  Inputs are
resident in HBM and larger than L2 (A ~0.95 GB, sinograms 0.54 GB).  `e2e` repeats the step
through the C-ABI from pinned host buffers (y, w up, image down).  `roofline` is the fused
update kernel's algorithmic HBM bytes over its own event-timed duration.

--impl reference: the repo's sequential C oracle (the only reference this paper has), timed
on the host cores on a bounded sample of the same per-update work.
"""
from __future__ import annotations

import argparse
import json
import math
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

MU_W = 0.02


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default="cfg4")
    ap.add_argument("--equits", type=float, default=6.0, help="equits per step")
    ap.add_argument("--batch-svs", type=int, default=0)
    ap.add_argument("--sv-side", type=int, default=0)
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-converge", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--no-psv", action="store_true", help="skip the PSV-ICD CPU comparison leg")
    ap.add_argument("--conv-iters", type=int, default=300, help="max iterations of a convergence run")
    return ap.parse_args()


# ----------------------------------------------------------------------------- clocks
class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled every 200 ms during the timed region."""
    Q = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap")

    def __init__(self, index):
        self.index = index
        self.lines = []
        self.p = None

    def __enter__(self):
        try:
            self.p = subprocess.Popen(["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.Q}",
                                       "--format=csv,noheader,nounits", "-lms", "200"],
                                      stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.p = None
        return self

    def _read(self):
        for line in self.p.stdout:
            self.lines.append(line.strip())

    def __exit__(self, *a):
        if self.p:
            self.p.terminate()
            try:
                self.p.wait(timeout=5)
            except Exception:
                self.p.kill()

    def summary(self):
        sm, mx, reasons = [], 0.0, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            f = [x.strip() for x in ln.split(",")]
            if len(f) < 7:
                continue
            try:
                sm.append(float(f[0]))
                mx = max(mx, float(f[1]))
            except ValueError:
                continue
            for n, v in zip(names, f[3:7]):
                if v.lower() == "active":
                    reasons.add(n)
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": mx or None,
                "reasons": sorted(reasons), "samples": len(sm)}


# ----------------------------------------------------------------------------- CPU oracle leg
def oracle_sample_setup():
    """Bounded sample of the workload's per-update work for the sequential oracle: a 128 x 128
    slice with config 4's pitch (dxy = 0.5 mm), 720 views and dc = dxy/2 (256 channels), so every
    voxel update touches ~2400 (view, channel) entries as at full size."""
    import oracle as O
    from synth import WorkloadConfig, make_case
    cfg = WorkloadConfig("cpu-sample", 128, 1, 720, 256, 9, 26, 0.005, fov=64.0)
    case = make_case(cfg, with_truth=False)
    og = O.Geometry(cfg.n, cfg.n, 1, cfg.dxy, cfg.nviews, cfg.nchannels, cfg.dchannel)
    A = O.sysmatrix(og)
    _, _, Aq = O.quantize(A)
    pr = O.Prior(sigma=cfg.sigma, nbhd=26)
    return O, og, Aq, pr, case, cfg


def oracle_time(O, og, Aq, pr, case, budget_s):
    x = np.zeros(og.nx * og.ny)
    e = O.error_sinogram(og, Aq, case.y.astype(np.float64), x)
    upd, t0, sweeps = 0, time.perf_counter(), 0
    while True:
        st, _ = O.icd_run(og, pr, Aq, case.w, x, e, 1, first_sweep=sweeps + 1, seed=3000)
        upd += st["updates"]
        sweeps += 1
        el = time.perf_counter() - t0
        if el >= budget_s:
            break
    return upd, el, sweeps


def cpu_baseline(budget_s=12.0):
    O, og, Aq, pr, case, cfg = oracle_sample_setup()
    upd, el, sweeps = oracle_time(O, og, Aq, pr, case, budget_s)
    return {"value": upd / el, "unit": "voxel updates/s", "cores": 1, "kind": "oracle",
            "sample": f"sequential C oracle (double), {sweeps} equits of a 128x128 slice at "
                      f"config-4 pitch (0.5 mm), 720 views x 256 channels (dc = dxy/2, "
                      f"{int(Aq.count.sum() / (cfg.n * cfg.n))} nnz/voxel), {upd} updates in {el:.1f} s"}


def psv_baseline(max_s=40.0, side=13):
    """The paper's CPU comparison system, PSV-ICD (Alg. 2; psvicd/, SURVEY 8(f)
    NEXT-4), on all host cores: time from the oracle's FBP image to < 10 HU RMSE against the
    committed cfg3 oracle golden on cfg3 (the paper's T1 workload shape), 20 % SV
    selection, SV side 13 (T1's PSV-ICD column).  A and the FBP image come from the oracle
    (test infrastructure; setup not timed).  The paper's 4.43x GPU-ICD / PSV-ICD is
    context only."""
    import oracle as O
    from psvicd import PSVICD
    from synth import CONFIGS, make_case
    t_setup = time.perf_counter()
    cfg = CONFIGS["cfg3"]
    case = make_case(cfg, 0, with_truth=False)
    og = O.Geometry(cfg.n, cfg.n, 1, cfg.dxy, cfg.nviews, cfg.nchannels, cfg.dchannel)
    _, _, Aq = O.quantize(O.sysmatrix(og))
    z = np.load(os.path.join(ROOT, "tests", "golden", "golden_cfg3.npz"))
    gold = z["x"].ravel().astype(np.float64)
    x = O.fbp(og, case.y).astype(np.float32).reshape(1, cfg.n, cfg.n).copy()
    e = O.error_sinogram(og, Aq, case.y.astype(np.float64), x.ravel().astype(np.float64))
    e = np.ascontiguousarray(e.astype(np.float32).reshape(case.y.shape))
    w = np.ascontiguousarray(case.w, np.float32)
    psv = PSVICD(cfg.n, cfg.n, 1, cfg.nviews, cfg.nchannels, Aq, sigma=cfg.sigma, nbhd=cfg.nbhd, sv_side=side)
    t_setup = time.perf_counter() - t_setup
    t, upd, hit, it, rm, nt = 0.0, 0, None, 0, None, None
    while t < max_s:
        st = psv.iterate(w, x, e, 1, frac=0.2)
        it += 1
        t += st["seconds"]
        upd += st["updates"]
        nt = st["threads"]
        rm = O.rmse_hu(x.ravel().astype(np.float64), gold)
        if rm < 10.0:
            hit = t
            break
    psv.close()
    return {"kind": "PSV-ICD (Alg. 2) on host threads", "workload": "cfg3: 512x512, 720 views x 1024 channels",
            "cores": nt, "sv_side": side, "frac": 0.2, "init": "oracle FBP (not timed)",
            "time_to_10hu_s": hit, "equits_to_10hu": upd / cfg.n ** 2 if hit else None, "iterations": it,
            "final_rmse_hu": rm, "updates_per_s": upd / t if t > 0 else None, "setup_s": t_setup}


def workload_config(cfg, side, args, world):
    """The `config` object of both arms (the reference arm times a bounded sample of it)."""
    sino_gb = 3 * cfg.nz * cfg.nviews * cfg.nchannels * 4 / 1e9
    return {"workload": f"{cfg.name}: {cfg.n}x{cfg.n}x{cfg.nz} volume, {cfg.nviews} views x "
                        f"{cfg.nchannels} channels parallel-beam 3-D Shepp-Logan, Poisson "
                        f"(lambda0=1e4), q-GGMRF {cfg.nbhd}-nbhd, SV side {side}",
            "equits_per_step": args.equits, "slab_slices_per_gpu": cfg.nz // world,
            "parallelism": f"z-slab x{world}", "batch_svs": args.batch_svs,
            "l2": "inputs larger than L2 (uint8 A ~1 GB + y, w, e %.2f GB, no flush needed)" % sino_gb}


def run_reference(args, rank, world):
    if rank != 0:
        return
    from synth import CONFIGS
    cfg_full = CONFIGS[args.config]
    O, og, Aq, pr, case, cfg = oracle_sample_setup()
    for _ in range(args.warmup):
        oracle_time(O, og, Aq, pr, case, 0.5)
    tot_u, tot_t = 0, 0.0
    for _ in range(args.steps):
        u, t, _ = oracle_time(O, og, Aq, pr, case, 3.0)
        tot_u += u
        tot_t += t
    v = tot_u / tot_t
    line = {"metric": "voxel updates/s", "value": v, "unit": "voxel updates/s", "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1000 * tot_t / args.steps,
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "f64",
            "data": "synthetic", "impl": "reference",
            "config": dict(workload_config(cfg_full, args.sv_side or cfg_full.sv_side, args, world),
                           sample="the oracle times a bounded sample with the workload's per-update work "
                                  "(a 128x128 slice at config-4 pitch, 720 views x 256 channels, 2396 "
                                  "nnz/voxel), not the whole cfg4 volume"),
            "cpu_baseline": {"value": v, "unit": "voxel updates/s", "cores": 1, "kind": "oracle",
                             "sample": "each step: >= 3 s of sequential-oracle equits on a bounded "
                                       "sample of the workload's per-update work: a 128x128 slice "
                                       "at config-4 pitch (0.5 mm), 720 views x 256 channels"},
            "e2e": {"value": v, "unit": "voxel updates/s", "h2d_bytes_per_step": 0,
                    "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# ----------------------------------------------------------------------------- convergence
def load_golden(config, y, w):
    """(x float32 [nz][n][n], meta) of the oracle golden of `config` if one exists for exactly this
    sinogram (hash check), else None.  Committed goldens live in tests/golden/, large ones in
    goldens/ (written by tools/make_golden.py, which calls only oracle/)."""
    from tools.make_golden import sino_hash
    for d in ("tests/golden", "goldens"):
        p = os.path.join(ROOT, d, f"golden_{config}.npz")
        if os.path.exists(p):
            z = np.load(p)
            meta = json.loads(str(z["meta"]))
            if meta.get("sino_sha") == sino_hash(y.cpu().numpy(), w.cpu().numpy()):
                return z["x"], {k: meta[k] for k in ("equits", "init", "selfconv_hu_last20", "order")} | {"file": os.path.relpath(p, ROOT)}
    return None


def converge(r, golden, init, stream, max_iter, target=10.0):
    """Iterate from `init` until RMSE-HU(x, golden) < target; device seconds of the iterations (and
    of mbir_init_fbp when init = fbp), equits, and the RMSE curve."""
    import torch
    f0, f1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    f0.record(stream)
    if init == "fbp":
        r.init_fbp()
    else:
        r.set_image(None)
    f1.record(stream)
    torch.cuda.synchronize()
    t = f0.elapsed_time(f1) / 1000.0
    eq, hist, hit = 0.0, [(0.0, round(r.rmse_hu(golden), 2))], None
    for it in range(max_iter):
        s = r.iterate(1)
        t += s["seconds"]
        eq += s["equits"]
        hist.append((round(eq, 3), round(r.rmse_hu(golden), 2)))
        if hist[-1][1] < target:
            hit = {"time_s": t, "equits": eq, "iterations": it + 1}
            break
    return {"time_to_10hu_s": hit["time_s"] if hit else None, "equits_to_10hu": hit["equits"] if hit else None,
            "iterations": len(hist) - 1, "final_rmse_hu": hist[-1][1], "init_s": f0.elapsed_time(f1) / 1000.0,
            "rmse_hu_curve": hist[:80]}


def converge_config(name, dev, stream, max_iter):
    import torch

    import paper_conf_ppopp_sabnewkbrm17_b200 as M
    from synth import CONFIGS, make_sinogram_torch
    cfg = CONFIGS[name]
    y, w = make_sinogram_torch(cfg, 0, dev)
    gz = load_golden(name, y, w)
    if gz is None:
        return {"golden": None}
    g = M.Geometry(cfg.n, cfg.n, cfg.nz, cfg.dxy, cfg.nviews, cfg.nchannels, cfg.dchannel)
    out = {"workload": f"{name}: {cfg.n}x{cfg.n}x{cfg.nz}, {cfg.nviews} views x {cfg.nchannels} channels",
           "golden": gz[1]}
    with M.Reconstructor(g, M.Prior(sigma=cfg.sigma, neighborhood=cfg.nbhd), M.Options(sv_side=cfg.sv_side),
                         device=dev.index or 0, stream=stream.cuda_stream) as r:
        r.set_sinogram(y, w)
        golden = torch.from_numpy(gz[0]).to(dev)
        converge(r, golden, "fbp", stream, 3)  # warm-up
        for init in ("fbp", "zero"):
            out["from_" + init] = converge(r, golden, init, stream, max_iter)
    return out


# ----------------------------------------------------------------------------- GPU leg
def main():
    args = parse()
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if args.impl == "reference":
        run_reference(args, rank, world)
        return

    import torch
    import torch.distributed as dist

    import paper_conf_ppopp_sabnewkbrm17_b200 as M
    from paper_conf_ppopp_sabnewkbrm17_b200 import dist as D
    from synth import CONFIGS, make_sinogram_torch

    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        dist.init_process_group("nccl", device_id=dev)
    cfg = CONFIGS[args.config]
    side = args.sv_side or cfg.sv_side
    nz = cfg.nz
    z0, nzl = D.slab(nz, world, rank)
    stream = torch.cuda.current_stream(dev)

    t_setup = time.perf_counter()
    y, w = make_sinogram_torch(cfg, 0, dev, z0, z0 + nzl)
    g = M.Geometry(cfg.n, cfg.n, nzl, cfg.dxy, cfg.nviews, cfg.nchannels, cfg.dchannel,
                   z_offset=z0, nz_total=nz)
    pr = M.Prior(sigma=cfg.sigma, neighborhood=cfg.nbhd)
    opt = M.Options(sv_side=side, batch_svs=args.batch_svs)
    nccl_id = D.broadcast_nccl_id() if world > 1 else None
    r = M.Reconstructor(g, pr, opt, device=local, stream=stream.cuda_stream, rank=rank,
                        nranks=world, nccl_id=nccl_id)
    r.set_sinogram(y, w)
    sizes = r.sizes()
    torch.cuda.synchronize()
    setup_s = time.perf_counter() - t_setup

    def barrier():
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()

    def allmax(v):
        if world == 1:
            return v
        t = torch.tensor([v], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())

    def step():
        r.set_image(None)  # x0 = 0, e = y (one forward kernel launch)
        return r.reconstruct(args.equits)

    for _ in range(args.warmup):
        step()
    barrier()
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    stats = []
    with ClockSampler(local) as clk:
        ev0.record(stream)
        for _ in range(args.steps):
            stats.append(step())
        ev1.record(stream)
        torch.cuda.synchronize()
    barrier()
    el = allmax(ev0.elapsed_time(ev1) / 1000.0)
    updates = sum(s["updates"] for s in stats)  # all-reduced over ranks by the library
    value = updates / el
    launches = sum(s["launches"] + 1 for s in stats)
    # ---- roofline of the fused update kernel (this rank's work / this rank's kernel time)
    nvox_plane = cfg.n * cfg.n
    nnz_avg = sizes["nnz"] / nvox_plane
    band_avg = sizes["band_entries"] / sizes["nsv"]
    ksec = sum(s["kernel_seconds"] for s in stats)
    klaunch = sum(s["kernel_launches"] for s in stats)
    local_updates = updates / world
    # SV-buffer traffic only for visits that updated something (fully zero-skipped ones move none)
    local_visits = sum(s["sv_visits"] - s["sv_visits_empty"] for s in stats) / world
    bytes_per_update = nnz_avg * 1 + cfg.nviews * 1 + 4  # u8 codes of the nnz, offsets, scale
    alg_bytes = local_updates * bytes_per_update + local_visits * 16 * band_avg
    achieved = alg_bytes / ksec / 1e9
    peaks = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json"))) if os.path.exists(
        os.path.join(ROOT, "MEASURED_PEAKS.json")) else {}
    peak = peaks.get("hbm_gbs", 6650.0)
    traffic = None
    tp = os.path.join(ROOT, "profiles", "icd_traffic.json")
    if os.path.exists(tp):
        tj = json.load(open(tp))
        traffic = tj.get("dram_bytes_per_update", 0) * local_updates / max(klaunch, 1)
    roof = {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
            "frac": achieved / peak, "traffic": traffic,
            "kernel": "k_svicd (fused SV update)", "kernel_share": ksec / el,
            "alg_bytes_per_update": alg_bytes / local_updates,
            "peak_source": "MEASURED_PEAKS.json hbm_gbs (copy)" if peaks else "fallback 6.65 TB/s"}

    # ---- end to end through the C-ABI with host buffers
    e2e = None
    if not args.no_e2e:
        yh = y.cpu().pin_memory()
        wh = w.cpu().pin_memory()
        xh = torch.empty((nzl, cfg.n, cfg.n), dtype=torch.float32).pin_memory()
        ke = max(1, min(args.steps, 3))
        barrier()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        upd_e = 0
        e0.record(stream)
        for _ in range(ke):
            r.set_sinogram(yh, wh)
            r.set_image(None)
            upd_e += r.reconstruct(args.equits)["updates"]
            r.image(xh)
        e1.record(stream)
        torch.cuda.synchronize()
        barrier()
        ele = allmax(e0.elapsed_time(e1) / 1000.0)
        e2e = {"value": upd_e / ele, "unit": "voxel updates/s",
               "h2d_bytes_per_step": int(2 * yh.numel() * 4 * world),
               "d2h_bytes_per_step": int(xh.numel() * 4 * world),
               "ms_per_step": 1000 * ele / ke}
        r.set_sinogram(y, w)

    # ---- time to converge (RMSE < 10 HU against the golden image of traditional ICD),
    # against the oracle's golden (tools/make_golden.py: sequential ICD from FBP until converged)
    # when one exists for this exact sinogram; device time of the iterations only (the per-
    # iteration RMSE reduction is outside it); from the FBP image (mbir_init_fbp, its time
    # counted) and from x0 = 0
    conv = None
    if not args.no_converge and world == 1:
        gz = load_golden(args.config, y, w)
        if gz is not None:
            golden = torch.from_numpy(gz[0]).to(dev)
            conv = {"golden": gz[1]}
            converge(r, golden, "fbp", stream, 3)  # warm-up (first FBP launch loads its module)
            for init in ("fbp", "zero"):
                conv["from_" + init] = converge(r, golden, init, stream, args.conv_iters)
        else:
            conv = {"golden": None, "note": "no oracle golden for this sinogram (tools/make_golden.py)"}
        # the paper's own workload (T1: 512^2, 720 views; GPU-ICD 0.407 s / 5.9 equits on
        # its data, context only) with the committed cfg3 golden
        if args.config != "cfg3":
            conv["cfg3"] = converge_config("cfg3", dev, stream, args.conv_iters)

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu:
        cpu = cpu_baseline()
    psv = None
    if rank == 0 and world == 1 and not args.no_psv and not args.no_cpu:
        psv = psv_baseline()
        g3 = ((conv or {}).get("cfg3") or {}).get("from_fbp") or {}
        if args.config == "cfg3":
            g3 = (conv or {}).get("from_fbp") or {}
        if psv.get("time_to_10hu_s") and g3.get("time_to_10hu_s"):
            psv["gpu_speedup_time_to_10hu"] = psv["time_to_10hu_s"] / g3["time_to_10hu_s"]

    if rank == 0:
        clocks = clk.summary()
        line = {
            "metric": "voxel updates/s", "value": value, "unit": "voxel updates/s",
            "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": 1000 * el / args.steps, "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": "f32 (A uint8)",
            "data": "synthetic",
            "config": workload_config(cfg, side, args, world),
            "updates_per_step": updates / args.steps,
            "time_to_converge": conv,
            "roofline": roof, "cpu_baseline": cpu, "psv_icd": psv, "e2e": e2e,
            "gpu_launches": launches, "clocks": clocks,
            "setup_s": setup_s, "sizes": sizes,
        }
        print(json.dumps(line), flush=True)
    r.close()
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
