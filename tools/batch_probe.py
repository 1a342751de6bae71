#!/usr/bin/env python
"""Convergence vs per-slice batch size on a 2-D case (asynchronous SV updates from x0 = 0):
iterations until RMSE < 10 HU against a deterministic-order (sequential) 100-equit golden."""
import argparse, os, sys
import numpy as np, torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ppopp_sabnewkbrm17_b200 as M
from synth import CONFIGS, make_case, sweep_configs
ap = argparse.ArgumentParser()
ap.add_argument("--case", default="sweep0")
ap.add_argument("--batches", default="0,8,16,32,64")
ap.add_argument("--golden-equits", type=float, default=100)
ap.add_argument("--zero-skip", type=int, default=1)
ap.add_argument("--det", type=int, default=0)
ap.add_argument("--fbp", type=int, default=0)
ap.add_argument("--cluster", type=int, default=0)
ap.add_argument("--max-equits", type=float, default=150)
a = ap.parse_args()
if a.case in CONFIGS:
    cfg, cid = CONFIGS[a.case], 0
else:
    cfg, cid = dict((c.name, (c, i)) for c, i in sweep_configs())[a.case]
c = make_case(cfg, cid, with_truth=False)
g = M.Geometry(cfg.n, cfg.n, cfg.nz, cfg.dxy, cfg.nviews, cfg.nchannels, cfg.dchannel)
pr = M.Prior(sigma=cfg.sigma, neighborhood=cfg.nbhd)
y, w = torch.from_numpy(c.y).cuda(), torch.from_numpy(c.w).cuda()
with M.Reconstructor(g, pr, M.Options(sv_side=cfg.sv_side, deterministic=1, zero_skip=0)) as r:
    r.set_sinogram(y, w)
    r.reconstruct(a.golden_equits)
    gold = torch.from_numpy(r.image().copy()).cuda()
print(cfg.name, cfg.n, cfg.nviews, "golden max", float(gold.max()))
for b in [int(x) for x in a.batches.split(",")]:
    with M.Reconstructor(g, pr, M.Options(sv_side=cfg.sv_side, batch_svs=b, batch_threshold=0, zero_skip=a.zero_skip, deterministic=a.det, cluster=a.cluster)) as r:
        r.set_sinogram(y, w)
        if a.fbp:
            r.init_fbp()
        t = eq = 0.0
        hist = []
        for it in range(400):
            st = r.iterate(1)
            t += st["seconds"]; eq += st["equits"]
            hu = r.rmse_hu(gold)
            if it < 4: hist.append(round(hu, 1))
            if hu < 10 or eq > a.max_equits: break
        print(f"batch {b:4d}: iters {it+1:4d} equits {eq:7.2f} device {t*1e3:8.2f} ms  final HU {hu:8.2f}  first HU {hist}")
