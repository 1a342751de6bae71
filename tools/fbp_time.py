#!/usr/bin/env python
"""Device time of mbir_init_fbp on cfg4 (FBP kernels + e = y - A x), three calls."""
import os, sys, torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ppopp_sabnewkbrm17_b200 as M
from synth import CONFIGS, make_sinogram_torch
cfg = CONFIGS["cfg4"]
y, w = make_sinogram_torch(cfg, 0, "cuda")
g = M.Geometry(cfg.n, cfg.n, cfg.nz, cfg.dxy, cfg.nviews, cfg.nchannels, cfg.dchannel)
with M.Reconstructor(g, M.Prior(sigma=cfg.sigma, neighborhood=26), M.Options(sv_side=9)) as r:
    r.set_sinogram(y, w)
    for i in range(3):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(); r.init_fbp(); e1.record(); torch.cuda.synchronize()
        print(f"init_fbp {i}: {e0.elapsed_time(e1):.1f} ms")
