#!/usr/bin/env python
"""Stage 2 of the config-5 sweep (BASELINE.json configs[4]): GPU time to converge on the cases
whose oracle golden tools/sweep_goldens.py has written (goldens/sweep/), and the speedup over the
sequential oracle's own time to converge on one host core -- the shape of the paper's headline
(611.79X over sequential ICD, 4.43X over 16-core PSV-ICD; context only: other data,
other hardware).

Both sides start from their FBP image (the oracle's and mbir_init_fbp, each timed) and stop at the
first iteration (GPU) / sweep (oracle) below 10 HU RMSE from the golden.  GPU time =
device time of init_fbp + the iterations (stats.seconds; the RMSE checks are outside it).  Also
reported: from x0 = 0.  Writes one JSON line per case and a summary (--out FILE)."""
import argparse
import glob
import json
import math
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ppopp_sabnewkbrm17_b200 as M  # noqa: E402
from synth import make_sinogram_torch, sweep_configs  # noqa: E402
from tools.make_golden import sino_hash  # noqa: E402


def run(r, golden, init, max_iter=400):
    s0, s1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    s0.record()
    if init == "fbp":
        r.init_fbp()
    else:
        r.set_image(None)
    s1.record()
    torch.cuda.synchronize()
    t, eq = s0.elapsed_time(s1) / 1e3, 0.0
    if r.rmse_hu(golden) < 10.0:
        return t, 0.0, 0
    for it in range(max_iter):
        st = r.iterate(1)
        t += st["seconds"]
        eq += st["equits"]
        if r.rmse_hu(golden) < 10.0:
            return t, eq, it + 1
    return None, eq, max_iter


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default=None)
    ap.add_argument("--set", default="main", choices=["main", "large"])
    a = ap.parse_args()
    allc = sweep_configs(40, 5001, sides=(11, 13), prefix="sweepL") if a.set == "large" else sweep_configs()
    pref = "sweepL" if a.set == "large" else "sweep"
    rows = []
    for path in sorted(glob.glob(os.path.join(ROOT, "goldens", "sweep", f"{pref}[0-9]*.npz"))):
        z = np.load(path)
        meta = json.loads(str(z["meta"]))
        cfg, cid = allc[meta["idx"]]
        y, w = make_sinogram_torch(cfg, cid, "cuda")
        if sino_hash(y.cpu().numpy(), w.cpu().numpy()) != meta["sino_sha"]:
            print(json.dumps({"case": cfg.name, "error": "sinogram differs from the golden's"}))
            continue
        golden = torch.from_numpy(z["x"]).cuda()
        g = M.Geometry(cfg.n, cfg.n, 1, cfg.dxy, cfg.nviews, cfg.nchannels, cfg.dchannel)
        try:
            r = M.Reconstructor(g, M.Prior(sigma=cfg.sigma, neighborhood=8), M.Options(sv_side=cfg.sv_side))
        except M.MbirError as ex:  # e.g. a side-13 SV buffer that neither one CTA nor a cluster holds
            row = {k: meta[k] for k in ("case", "n", "views", "sv_side")}
            row["unsupported"] = str(ex)
            rows.append(row)
            print(json.dumps(row), flush=True)
            continue
        with r:
            r.set_sinogram(y, w)
            run(r, golden, "fbp", 2)  # warm-up
            tf, ef, itf = run(r, golden, "fbp")
            tz, ez, itz = run(r, golden, "zero")
        row = {k: meta[k] for k in ("case", "phantom", "n", "views", "lambda0", "sv_side", "selfconv_hu_last20",
                                     "oracle_s_to_10hu", "oracle_equits_to_10hu")}
        row.update({"gpu_s_to_10hu": tf, "gpu_equits_to_10hu": ef, "gpu_iterations": itf,
                    "gpu_s_to_10hu_from_zero": tz, "gpu_equits_to_10hu_from_zero": ez,
                    "speedup": (meta["oracle_s_to_10hu"] / tf) if (tf and meta["oracle_s_to_10hu"]) else None})
        rows.append(row)
        print(json.dumps(row), flush=True)
    ok = [r_["speedup"] for r_ in rows if r_.get("speedup")]
    unsup = [r_ for r_ in rows if "unsupported" in r_]
    rows_run = [r_ for r_ in rows if "unsupported" not in r_]
    summary = {"cases": len(rows), "unsupported": len(unsup), "both_converged": len(ok),
               "geomean_speedup_vs_1core_oracle": math.exp(sum(math.log(s) for s in ok) / len(ok)) if ok else None,
               "min_speedup": min(ok) if ok else None, "max_speedup": max(ok) if ok else None,
               "gpu_equits_to_10hu_median": float(np.median([r_["gpu_equits_to_10hu"] for r_ in rows_run if r_["gpu_s_to_10hu"]])) if ok else None,
               "oracle_equits_to_10hu_median": float(np.median([r_["oracle_equits_to_10hu"] for r_ in rows_run if r_["oracle_equits_to_10hu"] is not None])) if rows_run else None,
               "oracle_cores": 1,
               "context": "paper: 611.79X geomean over sequential ICD, 4.43X over 16-core PSV-ICD (P:303), TO3 data, Titan X"}
    print(json.dumps(summary))
    if a.out:
        json.dump({"rows": rows, "summary": summary}, open(a.out, "w"), indent=1)


if __name__ == "__main__":
    main()
