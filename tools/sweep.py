#!/usr/bin/env python
"""BASELINE.json configs[4]: time-to-converge (< 10 HU RMSE) of the GPU path and of the sequential
C oracle on a bounded sample of the 200-case synthetic sweep (synth.sweep_configs: phantom incl.
baggage-like scenes, dose, view count, SV side; 2-D slices N in {128, 256}, M = 2N), and their
geometric-mean ratio -- the shape of the paper's headline (4.43X over 16 CPU cores).

Golden per case: 300 equits of the GPU path's deterministic mode without zero-skipping (exact
sequential ICD, the oracle's method; the MAP point is unique and the GPU/oracle parity of
converged images is pinned in tests/test_gpu_parity.py).  Both sides start from x0 = 0 with
zero-skipping and are stopped at the first iteration (GPU) / equit (oracle) below 10 HU.  GPU time
= device time of the update iterations (stats.seconds), RMSE checks excluded; oracle time = wall
clock of its sweeps on one host core (RMSE excluded).  The oracle is test infrastructure: this
tool, like bench.py's cpu_baseline, only times it.

usage: python tools/sweep.py [--cases 8] [--stride 25] [--oracle-cap 90] [--out FILE]"""
import argparse
import json
import math
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle as O  # noqa: E402
import paper_conf_ppopp_sabnewkbrm17_b200 as M  # noqa: E402
from synth import make_case, sweep_configs  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--cases", type=int, default=8)
ap.add_argument("--stride", type=int, default=25, help="take every stride-th case of the 200")
ap.add_argument("--oracle-cap", type=float, default=90.0, help="max oracle seconds per case")
ap.add_argument("--out", default=None)
ap.add_argument("--golden-equits", type=float, default=300.0)
a = ap.parse_args()

cases = sweep_configs()[:: a.stride][: a.cases]
rows = []
for cfg, cid in cases:
    c = make_case(cfg, cid, with_truth=False)
    g = M.Geometry(cfg.n, cfg.n, 1, cfg.dxy, cfg.nviews, cfg.nchannels, cfg.dchannel)
    pr = M.Prior(sigma=cfg.sigma, neighborhood=8)
    y = torch.from_numpy(c.y).cuda()
    w = torch.from_numpy(c.w).cuda()
    with M.Reconstructor(g, pr, M.Options(sv_side=cfg.sv_side, deterministic=1, zero_skip=0)) as r:
        r.set_sinogram(y, w)
        r.reconstruct(a.golden_equits)
        golden = r.image().copy()
    gold_t = torch.from_numpy(golden).cuda()
    with M.Reconstructor(g, pr, M.Options(sv_side=cfg.sv_side)) as r:
        r.set_sinogram(y, w)
        t_gpu, eq_gpu, hu = 0.0, 0.0, 1e9
        for _ in range(2000):
            st = r.iterate(1)
            t_gpu += st["seconds"]
            eq_gpu += st["equits"]
            hu = r.rmse_hu(gold_t)
            if hu < 10.0:
                break
    og = O.Geometry(cfg.n, cfg.n, 1, cfg.dxy, cfg.nviews, cfg.nchannels, cfg.dchannel)
    _, _, Aq = O.quantize(O.sysmatrix(og))
    opr = O.Prior(sigma=cfg.sigma, nbhd=8)
    x = np.zeros(cfg.n * cfg.n)
    e = O.error_sinogram(og, Aq, c.y.astype(np.float64), x)
    t_orc, eq_orc, ohu, done = 0.0, 0, 1e9, False
    gflat = golden.ravel().astype(np.float64)
    while t_orc < a.oracle_cap:
        t0 = time.perf_counter()
        O.icd_run(og, opr, Aq, c.w, x, e, 1, first_sweep=eq_orc + 1, seed=3000, zero_skip=True)
        t_orc += time.perf_counter() - t0
        eq_orc += 1
        ohu = O.rmse_hu(x, gflat)
        if ohu < 10.0:
            done = True
            break
    row = {"case": cfg.name, "phantom": cfg.phantom, "case_id": cid, "n": cfg.n, "views": cfg.nviews,
           "lambda0": cfg.lambda0, "sv_side": cfg.sv_side, "gpu_s": t_gpu, "gpu_equits": eq_gpu,
           "oracle_s": t_orc, "oracle_equits": eq_orc, "oracle_converged": done,
           "speedup": t_orc / t_gpu if t_gpu > 0 else None}
    rows.append(row)
    print(json.dumps(row), flush=True)
ok = [r_["speedup"] for r_ in rows if r_["oracle_converged"] and r_["speedup"]]
summary = {"cases": len(rows), "converged_cases": len(ok),
           "geomean_speedup_vs_1core_oracle": math.exp(sum(math.log(s) for s in ok) / len(ok)) if ok else None,
           "oracle_cores": 1, "note": "bounded sample of synth.sweep_configs(); golden = GPU deterministic (sequential) ICD, no zero-skip, %g equits" % a.golden_equits}
print(json.dumps(summary))
if a.out:
    json.dump({"rows": rows, "summary": summary}, open(a.out, "w"), indent=1)
