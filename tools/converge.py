#!/usr/bin/env python
"""Time to converge against the oracle golden (RMSE < 10 HU vs traditional ICD's image;
tools/make_golden.py): per iteration device time, equits and RMSE-HU of the GPU path for a config,
an initial image (x0 = 0 or FBP) and a batching choice.  Prints one JSON line per run."""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ppopp_sabnewkbrm17_b200 as M  # noqa: E402
from synth import CONFIGS, make_sinogram_torch  # noqa: E402
from tools.make_golden import sino_hash  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="cfg3")
    ap.add_argument("--golden", default="")
    ap.add_argument("--init", default="fbp", choices=["fbp", "zero"])
    ap.add_argument("--batch-svs", type=int, default=0)
    ap.add_argument("--zero-skip", type=int, default=1)
    ap.add_argument("--period", type=int, default=4)
    ap.add_argument("--iters", type=int, default=60)
    ap.add_argument("--target", type=float, default=10.0)
    ap.add_argument("--sv-side", type=int, default=0)
    ap.add_argument("--det", type=int, default=0)
    ap.add_argument("--sweep", type=int, default=-1, help="a config-5 case index (golden from goldens/sweep/)")
    a = ap.parse_args()
    cid = 0
    if a.sweep >= 0:
        from synth import sweep_configs
        cfg, cid = sweep_configs()[a.sweep]
        a.config = cfg.name
        gpath = os.path.join(ROOT, "goldens", "sweep", f"{cfg.name}.npz")
    else:
        cfg = CONFIGS[a.config]
        gpath = a.golden or os.path.join(ROOT, "tests", "golden", f"golden_{a.config}.npz")
    gz = np.load(gpath)
    meta = json.loads(str(gz["meta"]))
    y, w = make_sinogram_torch(cfg, cid, "cuda")
    if sino_hash(y.cpu().numpy(), w.cpu().numpy()) != meta["sino_sha"]:
        raise SystemExit("golden was computed for a different sinogram")
    golden = torch.from_numpy(gz["x"]).cuda()
    g = M.Geometry(cfg.n, cfg.n, cfg.nz, cfg.dxy, cfg.nviews, cfg.nchannels, cfg.dchannel)
    opt = M.Options(sv_side=a.sv_side or cfg.sv_side, batch_svs=a.batch_svs,
                    batch_threshold=0 if a.batch_svs else -1, zero_skip=a.zero_skip,
                    zero_skip_period=a.period, deterministic=a.det)
    with M.Reconstructor(g, M.Prior(sigma=cfg.sigma, neighborhood=cfg.nbhd), opt) as r:
        r.set_sinogram(y, w)
        for rep in range(1 if a.det else 2):  # rep 0 warms up
            s0, s1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            s0.record()
            if a.init == "fbp":
                r.init_fbp()
            else:
                r.set_image(None)
            s1.record()
            torch.cuda.synchronize()
            t, eq = s0.elapsed_time(s1) / 1e3, 0.0
            hist = [(0.0, 0.0, round(r.rmse_hu(golden), 2))]
            hit = None
            for it in range(a.iters):
                st = r.iterate(1)
                t += st["seconds"]
                eq += st["equits"]
                hist.append((round(t, 5), round(eq, 3), round(r.rmse_hu(golden), 2)))
                if hit is None and hist[-1][2] < a.target:
                    hit = {"time_s": t, "equits": eq, "iterations": it + 1}
        print(json.dumps({"config": a.config, "init": a.init, "batch_svs": a.batch_svs, "det": a.det,
                          "zero_skip": a.zero_skip, "period": a.period, "to_target": hit,
                          "target_hu": a.target, "golden": {k: meta.get(k) for k in ("equits", "golden_equits", "selfconv_hu_last20", "init")},
                          "final_hu": hist[-1][2], "curve": hist}))


if __name__ == "__main__":
    main()
