#!/usr/bin/env python
"""Per-iteration timing of the GPU path on a config: updates, SV visits, device time and
update-kernel time per iteration (diagnostic for where the time goes)."""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import paper_conf_ppopp_sabnewkbrm17_b200 as M  # noqa: E402
from synth import CONFIGS, make_sinogram_torch  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="cfg4")
ap.add_argument("--iters", type=int, default=12)
ap.add_argument("--zero-skip", type=int, default=1)
ap.add_argument("--sv-side", type=int, default=0)
ap.add_argument("--batch-svs", type=int, default=0)
ap.add_argument("--cluster", type=int, default=0)
ap.add_argument("--quantize", type=int, default=1)
ap.add_argument("--vps", type=int, default=0, help="voxels_per_step (0 auto)")
a = ap.parse_args()
cfg = CONFIGS[a.config]
y, w = make_sinogram_torch(cfg, 0, "cuda")
g = M.Geometry(cfg.n, cfg.n, cfg.nz, cfg.dxy, cfg.nviews, cfg.nchannels, cfg.dchannel)
r = M.Reconstructor(g, M.Prior(sigma=cfg.sigma, neighborhood=cfg.nbhd),
                    M.Options(sv_side=a.sv_side or cfg.sv_side, zero_skip=a.zero_skip,
                              batch_svs=a.batch_svs, cluster=a.cluster, quantize_A=a.quantize,
                              voxels_per_step=a.vps))
import time  # noqa: E402
for k in range(2):
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    r.set_sinogram(y, w)
    torch.cuda.synchronize()
    print(f"set_sinogram {k} {(time.perf_counter() - t0) * 1e3:.2f} ms")
print(json.dumps(r.sizes()))
for rep in range(2):
    r.set_image(None)
    for it in range(a.iters):
        s = r.iterate(1)
        if rep == 1 or it == 0:
            print(f"{'iter' if rep else 'first'} {it + 1:3d} upd {s['updates']:10d} skip {s['skipped']:10d} visits {s['sv_visits']:7d} "
                  f"t {s['seconds'] * 1e3:8.2f} ms  kernel {s['kernel_seconds'] * 1e3:8.2f} ms  "
                  f"ns/upd {1e9 * s['kernel_seconds'] / max(s['updates'], 1):7.2f}  "
                  f"us/visit {1e6 * s['kernel_seconds'] / max(s['sv_visits'], 1) * 148:8.2f}")
r.close()
