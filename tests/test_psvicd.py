"""PSV-ICD CPU comparison build (Alg. 2) against the oracle.

CPU-only.  Pins: with one SV covering the slice, one thread and raster order, one PSV-ICD
iteration IS a sequential ICD sweep in raster order (Alg. 2 with a single SV reduces to Alg. 1
applied voxel by voxel), so it equals the oracle's sweep with that order; with SVs updated in
parallel on host threads (any order, top-20 % / random-20 % selection, zero-skip with reading R9's
re-admission) it converges to the unique MAP the oracle converges to (1 HU / 1e-4 cost, the
north-star parity bar), and its error sinogram stays e = y - A x."""
import numpy as np
import pytest

import oracle as O
from psvicd import PSVICD
from synth import CONFIGS, WorkloadConfig, make_case


@pytest.fixture(scope="module")
def cfg1():
    cfg = CONFIGS["cfg1"]
    case = make_case(cfg)
    og = O.Geometry(cfg.n, cfg.n, 1, cfg.dxy, cfg.nviews, cfg.nchannels, cfg.dchannel)
    A = O.sysmatrix(og)
    _, _, Aq = O.quantize(A)
    return cfg, case, og, Aq


def _start(og, Aq, case):
    x = np.zeros((og.nz, og.ny, og.nx), np.float32)
    e = O.error_sinogram(og, Aq, case.y.astype(np.float64), x.astype(np.float64)).astype(np.float32)
    return x, e.reshape(case.y.shape)


def test_single_sv_raster_is_sequential_icd(cfg1):
    cfg, case, og, Aq = cfg1
    psv = PSVICD(cfg.n, cfg.n, 1, cfg.nviews, cfg.nchannels, Aq, sigma=cfg.sigma, nbhd=8, sv_side=cfg.n)
    x, e = _start(og, Aq, case)
    w = np.ascontiguousarray(case.w, np.float32)
    for it in range(3):
        psv.iterate(w, x, e, 1, frac=1.0, zero_skip=False, threads=1, raster=True)
    xo = np.zeros(cfg.n * cfg.n)
    eo = O.error_sinogram(og, Aq, case.y.astype(np.float64), xo)
    O.icd_run(og, O.Prior(sigma=cfg.sigma, nbhd=8), Aq, case.w, xo, eo, 3, zero_skip=False,
              order=np.arange(cfg.n * cfg.n))
    rel = np.abs(x.ravel() - xo).max() / np.abs(xo).max()
    assert rel < 2e-4, rel
    assert np.abs(e.ravel() - eo.ravel()).max() < 1e-4 * np.abs(case.y).max()


@pytest.mark.parametrize("side,zero_skip", [(9, True), (13, True), (5, False)])
def test_parallel_psv_converges_to_oracle_map(cfg1, side, zero_skip):
    cfg, case, og, Aq = cfg1
    pr = O.Prior(sigma=cfg.sigma, nbhd=8)
    xo = np.zeros(cfg.n * cfg.n)
    eo = O.error_sinogram(og, Aq, case.y.astype(np.float64), xo)
    O.icd_run(og, pr, Aq, case.w, xo, eo, 150, seed=3000, zero_skip=False)
    psv = PSVICD(cfg.n, cfg.n, 1, cfg.nviews, cfg.nchannels, Aq, sigma=cfg.sigma, nbhd=8, sv_side=side)
    x, e = _start(og, Aq, case)
    w = np.ascontiguousarray(case.w, np.float32)
    st = psv.iterate(w, x, e, 600, frac=0.2, zero_skip=zero_skip, threads=4)
    assert st["updates"] > 100 * cfg.n * cfg.n
    xg = x.ravel().astype(np.float64)
    rm = O.rmse_hu(xg, xo)
    assert rm < 1.0, rm
    cg = O.cost(og, pr, Aq, case.y, case.w, xg)
    co = O.cost(og, pr, Aq, case.y, case.w, xo)
    assert abs(cg - co) <= 1e-4 * abs(co), (cg, co)
    ee = O.error_sinogram(og, Aq, case.y.astype(np.float64), xg)
    assert np.abs(e.ravel() - ee.ravel()).max() < 1e-3 * np.abs(case.y).max()


def test_parallel_psv_3d_converges_to_oracle_map():
    cfg = WorkloadConfig("mini3d", 40, 4, 60, 64, 7, 26, 0.002)
    case = make_case(cfg)
    og = O.Geometry(cfg.n, cfg.n, cfg.nz, cfg.dxy, cfg.nviews, cfg.nchannels, cfg.dchannel)
    A = O.sysmatrix(og)
    _, _, Aq = O.quantize(A)
    pr = O.Prior(sigma=cfg.sigma, nbhd=26)
    xo = np.zeros(cfg.n * cfg.n * cfg.nz)
    eo = O.error_sinogram(og, Aq, case.y.astype(np.float64), xo)
    O.icd_run(og, pr, Aq, case.w, xo, eo, 150, seed=3000, zero_skip=False)
    psv = PSVICD(cfg.n, cfg.n, cfg.nz, cfg.nviews, cfg.nchannels, Aq, sigma=cfg.sigma, nbhd=26, sv_side=7)
    x, e = _start(og, Aq, case)
    w = np.ascontiguousarray(case.w, np.float32)
    psv.iterate(w, x, e, 600, frac=0.2, threads=4)
    xg = x.ravel().astype(np.float64)
    assert O.rmse_hu(xg, xo) < 1.0
    cg = O.cost(og, pr, Aq, case.y, case.w, xg)
    co = O.cost(og, pr, Aq, case.y, case.w, xo)
    assert abs(cg - co) <= 1e-4 * abs(co), (cg, co)


def test_psv_rejects_bad_arguments(cfg1):
    cfg, case, og, Aq = cfg1
    with pytest.raises(ValueError):
        PSVICD(cfg.n, cfg.n, 1, cfg.nviews, cfg.nchannels, Aq, sigma=cfg.sigma, nbhd=7)
    psv = PSVICD(cfg.n, cfg.n, 1, cfg.nviews, cfg.nchannels, Aq, sigma=cfg.sigma, nbhd=8, sv_side=9)
    x, e = _start(og, Aq, case)
    w = np.ascontiguousarray(case.w, np.float32)
    with pytest.raises(RuntimeError):
        psv.iterate(w, x, e, 1, frac=0.0)
