#!/usr/bin/env python
"""Stage 1 of the config-5 sweep (BASELINE.json configs[4]; tools/sweep.py is stage 2): for each
selected case of synth.sweep_configs(), the oracle's golden and the oracle's own time to converge.

Calls only oracle/ and synth/: x0 = the oracle's FBP (clipped at 0), then sequential ICD without
zero-skipping (random order per sweep) for E sweeps on ONE host thread, every iterate kept.
golden = x_E (self-convergence RMSE(x_{E-20}, x_E) recorded, must be < 0.1 HU); the oracle's
time-to-10 HU = its cumulative sweep time (FBP included) at the first sweep whose iterate
is < 10 HU from the golden.  Writes goldens/sweep/<case>.npz and appends one JSON line per case
to goldens/sweep/oracle.jsonl.

  python tools/sweep_goldens.py --cases 0,4,8,...   (indices into sweep_configs())
  python tools/sweep_goldens.py --set large --cases all --jobs 32   (the side-11/13 supplement,
                                                                    one process per case)
"""
import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import oracle as O  # noqa: E402
from synth import make_case, sweep_configs  # noqa: E402
from tools.make_golden import sino_hash  # noqa: E402


def case_set(name):
    """the 200-case config-5 sample, or the side-11/13 supplement"""
    return sweep_configs(40, 5001, sides=(11, 13), prefix="sweepL") if name == "large" else sweep_configs()


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--cases", required=True, help="comma-separated indices, or 'all'")
    ap.add_argument("--equits", type=int, default=60)
    ap.add_argument("--set", default="main", choices=["main", "large"])
    ap.add_argument("--jobs", type=int, default=1, help="cases run in parallel processes")
    a = ap.parse_args()
    allc = case_set(a.set)
    idxs = list(range(len(allc))) if a.cases == "all" else [int(v) for v in a.cases.split(",") if v]
    if a.jobs > 1:
        import subprocess
        procs = []
        for i, idx in enumerate(idxs):
            procs.append(subprocess.Popen([sys.executable, os.path.abspath(__file__), "--cases", str(idx),
                                           "--equits", str(a.equits), "--set", a.set]))
            if len(procs) >= a.jobs:
                procs.pop(0).wait()
        for pr_ in procs:
            pr_.wait()
        return
    out = os.path.join(ROOT, "goldens", "sweep")
    os.makedirs(out, exist_ok=True)
    for idx in idxs:
        cfg, cid = allc[idx]
        path = os.path.join(out, f"{cfg.name}.npz")
        if os.path.exists(path):
            continue
        case = make_case(cfg, cid, with_truth=False)
        og = O.Geometry(cfg.n, cfg.n, 1, cfg.dxy, cfg.nviews, cfg.nchannels, cfg.dchannel)
        _, _, Aq = O.quantize(O.sysmatrix(og))
        pr = O.Prior(sigma=cfg.sigma, nbhd=8)
        t0 = time.perf_counter()
        x = O.fbp(og, case.y).ravel().copy()
        e = O.error_sinogram(og, Aq, case.y.astype(np.float64), x)
        times, its = [time.perf_counter() - t0], [x.copy()]
        for s in range(1, a.equits + 1):
            t1 = time.perf_counter()
            O.icd_run(og, pr, Aq, case.w, x, e, 1, first_sweep=s, seed=7000, zero_skip=False)
            times.append(times[-1] + time.perf_counter() - t1)
            its.append(x.copy())
        gold = its[-1]
        hu = [O.rmse_hu(v, gold) for v in its]
        k10 = next((k for k, h in enumerate(hu) if h < 10.0), None)
        row = {"idx": idx, "case": cfg.name, "phantom": cfg.phantom, "case_id": cid, "n": cfg.n,
               "views": cfg.nviews, "lambda0": cfg.lambda0, "sv_side": cfg.sv_side, "sigma": cfg.sigma,
               "golden_equits": a.equits, "selfconv_hu_last20": hu[a.equits - 20],
               "oracle_s_to_10hu": times[k10] if k10 is not None else None,
               "oracle_equits_to_10hu": k10, "oracle_fbp_s": times[0], "oracle_cores": 1,
               "sino_sha": sino_hash(case.y, case.w)}
        np.savez_compressed(path, x=gold.reshape(1, cfg.n, cfg.n).astype(np.float32), meta=json.dumps(row))
        with open(os.path.join(out, "oracle.jsonl"), "a") as f:
            f.write(json.dumps(row) + "\n")
        print(json.dumps(row), flush=True)


if __name__ == "__main__":
    main()
