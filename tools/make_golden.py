#!/usr/bin/env python
"""Golden image for time-to-converge ("the golden output image [from] the traditional ICD
algorithm for 40 equits, by when it is known to converge"; reading R11).

Calls only oracle/ (and the seeded input generator synth/): x0 = the oracle's textbook FBP of y
(clipped at 0), then sequential ICD without zero-skipping (the MAP estimate it converges to is
unique) in slice-parity halves on host threads (oracle.icd_run_zpar, an exact serialisation of
sequential ICD), random order per sweep.  Runs E equits and records the self-convergence
RMSE(x_{E-20}, x_E), which must be < 0.1 HU for the golden to be used (reading R11).

  python tools/make_golden.py --config cfg3 --equits 100
writes tests/golden/golden_<config>.npz (x float32 [nz][n][n] + metadata incl. a hash of the
sinogram it was computed for, which bench.py checks before using it).
"""
import argparse
import hashlib
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import oracle as O  # noqa: E402
from synth import CONFIGS, make_case  # noqa: E402


def sino_hash(y, w):
    h = hashlib.sha256()
    h.update(np.ascontiguousarray(y, np.float32).tobytes())
    h.update(np.ascontiguousarray(w, np.float32).tobytes())
    return h.hexdigest()[:16]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="cfg3")
    ap.add_argument("--equits", type=int, default=100)
    ap.add_argument("--threads", type=int, default=0)
    ap.add_argument("--out", default="")
    ap.add_argument("--resume", default="", help="continue from this golden file's image (sweeps numbered on)")
    a = ap.parse_args()
    cfg = CONFIGS[a.config]
    t0 = time.time()
    case = make_case(cfg, 0, with_truth=False)
    og = O.Geometry(cfg.n, cfg.n, cfg.nz, cfg.dxy, cfg.nviews, cfg.nchannels, cfg.dchannel)
    A = O.sysmatrix(og)
    _, _, Aq = O.quantize(A)  # the uint8 A the GPU path runs with
    pr = O.Prior(sigma=cfg.sigma, nbhd=cfg.nbhd)
    first = 1
    if a.resume:
        z0 = np.load(a.resume)
        m0 = json.loads(str(z0["meta"]))
        assert m0["sino_sha"] == sino_hash(case.y, case.w)
        x = z0["x"].ravel().astype(np.float64).copy()
        first = m0["equits"] + 1
    else:
        x = O.fbp(og, case.y).ravel().copy()
    e = O.error_sinogram(og, Aq, case.y.astype(np.float64), x)
    print(f"setup {time.time() - t0:.0f} s", flush=True)
    hist, prev = [], None
    for s in range(1, a.equits + 1):
        O.icd_run_zpar(og, pr, Aq, case.w, x, e, 1, first_sweep=first + s - 1, seed=7000, zero_skip=False,
                       threads=a.threads or None)
        if s == a.equits - 20:
            prev = x.copy()
        if s % 10 == 0:
            print(f"equit {s}  {time.time() - t0:.0f} s", flush=True)
    selfconv = O.rmse_hu(prev, x) if prev is not None else None
    meta = {"config": a.config, "case_id": 0, "init": "oracle FBP (clipped at 0)", "equits": first - 1 + a.equits,
            "order": "random per sweep and slice, slice-parity halves (oracle.icd_run_zpar), seed 7000",
            "zero_skip": False, "A": "uint8 codes (oracle.quantize)", "sigma": cfg.sigma, "nbhd": cfg.nbhd,
            "selfconv_hu_last20": selfconv, "sino_sha": sino_hash(case.y, case.w),
            "seconds": time.time() - t0}
    out = a.out or os.path.join(ROOT, "tests", "golden", f"golden_{a.config}.npz")
    np.savez_compressed(out, x=x.reshape(cfg.nz, cfg.n, cfg.n).astype(np.float32), meta=json.dumps(meta))
    print(json.dumps(meta))


if __name__ == "__main__":
    main()
