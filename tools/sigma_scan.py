#!/usr/bin/env python
"""sigma_x scan on one config (reading R21): for each sigma, exact sequential SV-ICD
(deterministic mode, one CTA) from the FBP image for E sweeps; reports the RMSE-HU of the result
to the phantom (pixel-averaged truth), the self-convergence RMSE(x_{E/2}, x_E) and the curve of
RMSE to the final image.  The sigma minimising RMSE-to-phantom is the reconstruction a user would
pick."""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ppopp_sabnewkbrm17_b200 as M  # noqa: E402
from synth import CONFIGS, make_sinogram_torch, phantom_image, slice_ellipses  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="cfg3")
ap.add_argument("--sigmas", default="0.0015,0.002,0.003,0.005")
ap.add_argument("--sweeps", type=int, default=80)
ap.add_argument("--det", type=int, default=1)
a = ap.parse_args()
cfg = CONFIGS[a.config]
y, w = make_sinogram_torch(cfg, 0, "cuda")
truth = np.stack([phantom_image(slice_ellipses(cfg, z, 1000), cfg.n) for z in range(cfg.nz)]).astype(np.float32)
g = M.Geometry(cfg.n, cfg.n, cfg.nz, cfg.dxy, cfg.nviews, cfg.nchannels, cfg.dchannel)
for s in [float(v) for v in a.sigmas.split(",")]:
    with M.Reconstructor(g, M.Prior(sigma=s, neighborhood=cfg.nbhd),
                         M.Options(sv_side=cfg.sv_side, deterministic=a.det, zero_skip=0)) as r:
        r.set_sinogram(y, w)
        r.init_fbp()
        fbp_truth = r.rmse_hu(truth)
        imgs = []
        for k in range(a.sweeps):
            r.iterate(1)
            if (k + 1) in (1, 2, 3, 5, 8, 12, 20, 30, 40, a.sweeps // 2, a.sweeps):
                imgs.append((k + 1, r.image().copy()))
        fin = imgs[-1][1]
        curve = [(k, round(float(1000 * np.sqrt(np.mean((im.astype(np.float64) - fin) ** 2)) / 0.02), 2)) for k, im in imgs]
        print(json.dumps({"sigma": s, "fbp_to_truth": fbp_truth, "map_to_truth": r.rmse_hu(truth),
                          "zeros": float((fin == 0).mean()), "curve_to_final": curve}), flush=True)
