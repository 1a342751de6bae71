"""GPU parity: the CUDA path (through the C-ABI) against the sequential C oracle on the same
seeded inputs (BASELINE.json north_star tolerances):
  - system matrix integer index structure and uint8 codes bit-exact, values to fp32 rounding;
  - theta1, theta2, delta at a fixed state within 1e-5 (reading R20's normalisation);
  - deterministic-order updates track the sequential oracle update by update;
  - converged image within 1 HU RMSE and MAP cost within 1e-4 relative of the oracle's.
"""
import numpy as np
import pytest

import oracle as O
import paper_conf_ppopp_sabnewkbrm17_b200 as M
from synth import CONFIGS, WorkloadConfig, make_case
from tests.helpers import deterministic_order, geoms

pytestmark = pytest.mark.gpu

MU_W = 0.02


@pytest.fixture(scope="module")
def cfg1():
    cfg = CONFIGS["cfg1"]
    case = make_case(cfg)
    g, og = geoms(cfg)
    A = O.sysmatrix(og)
    codes, amax, Aq = O.quantize(A)
    return cfg, case, g, og, A, codes, amax, Aq


def small3d():
    """A 3-D case small enough for the oracle: 40 x 40 x 4 slices, 26-neighbourhood."""
    return WorkloadConfig("mini3d", 40, 4, 60, 64, 7, 26, 0.002)


# ------------------------------------------------------------------ system matrix (a1)
@pytest.mark.parametrize("quant", [1, 0])
def test_sysmatrix_bit_exact_index_structure(cfg1, quant):
    cfg, case, g, og, A, codes, amax, Aq = cfg1
    with M.Reconstructor(g, M.Prior(neighborhood=8), M.Options(sv_side=cfg.sv_side, quantize_A=quant)) as r:
        first, count, vals, gcodes, scales = r.sysmatrix()
        sz = r.sizes()
    np.testing.assert_array_equal(count, A.count)
    m = A.count > 0
    np.testing.assert_array_equal(first[m], A.first[m])
    assert sz["nnz"] == int(A.count.sum())
    if quant:
        # the buffers the update kernel reads: codes bit-exact, scale = fp32(amax/255), and the
        # exported values are the dequantised code * scale it computes with
        np.testing.assert_array_equal(gcodes, codes)
        np.testing.assert_array_equal(scales, (amax / 255).astype(np.float32))
        np.testing.assert_array_equal(vals, codes.astype(np.float32) * scales[:, None, None])
        np.testing.assert_allclose(vals, Aq.vals, rtol=2.5e-7, atol=0)
    else:
        # the stored fp32 values (read back from the buffer the kernel uses) against the oracle's
        # polygon-clipping areas: two double-precision formulations of the same strip integral,
        # each rounded once to fp32 (R5): within 1 ulp of fp32 of the value, plus an
        # absolute term for near-empty sliver entries, whose double-precision difference is
        # dominated by cancellation in either formulation (measured <= 1e-13 of the column max)
        d = np.abs(vals.astype(np.float64) - A.vals)
        ulp = np.spacing(np.abs(A.vals).astype(np.float32)).astype(np.float64)
        amaxc = A.vals.max(axis=(1, 2), keepdims=True)
        print("max |dA| / ulp:", (d / np.maximum(ulp, 1e-45)).max(), " max |dA| / column max:", (d / amaxc).max())
        assert np.all(d <= ulp + 1e-12 * amaxc)


def test_sysmatrix_paper_geometry_sampled():
    """Config-3 geometry (512^2, 720 views, 1024 channels) in the launch configuration the
    bench uses: the full A is too large to export, so 256 sampled voxels' columns (including
    the image corners, which lose views off the detector) are compared with the oracle's."""
    cfg = CONFIGS["cfg3"]
    g, og = geoms(cfg)
    rng = np.random.default_rng(3)
    vox = np.concatenate([rng.integers(0, cfg.n * cfg.n, 252), [0, cfg.n - 1, cfg.n * (cfg.n - 1),
                                                                cfg.n * cfg.n - 1]])
    with M.Reconstructor(g, M.Prior(neighborhood=8), M.Options(sv_side=cfg.sv_side)) as r:
        first, count, vals, gcodes, scales = r.sysmatrix_columns(vox)
        sz = r.sizes()
    assert sz["svb_rows"] <= 32
    for q, j in enumerate(vox):
        ix, iy = int(j % cfg.n), int(j // cfg.n)
        f, c, v, mc = O.sysmatrix_column(og, ix, iy, K=4)
        assert mc <= 4
        np.testing.assert_array_equal(count[q], c)
        np.testing.assert_array_equal(first[q][c > 0], f[c > 0])
        cd, am = O.quantize_column(v, c)
        np.testing.assert_array_equal(gcodes[q], cd)
        assert scales[q] == np.float32(am / 255)
        np.testing.assert_array_equal(vals[q], cd.astype(np.float32) * scales[q])


# ------------------------------------------------------------------ fixed-state probe (a4, a5)
def _fixed_state(cfg, case, og, Aq, pr, sweeps=3):
    x = np.zeros(og.nx * og.ny * og.nz)
    e = O.error_sinogram(og, Aq, case.y.astype(np.float64), x)
    O.icd_run(og, pr, Aq, case.w, x, e, sweeps, seed=5)
    x32 = x.astype(np.float32)
    e = O.error_sinogram(og, Aq, case.y.astype(np.float64), x32.astype(np.float64))
    return x32, e


def _check_probe(og, pr, Aq, case, x32, e, t1g, t2g, dg, vox):
    plane = og.nx * og.ny
    for q, j in enumerate(vox):
        xx = x32.astype(np.float64).copy()
        t1, t2, dl = O.voxel_update(og, pr, Aq, case.w, xx, e.copy(), int(j), apply=False)
        jj = j % plane
        z = j // plane
        k = np.arange(og.nviews)[:, None]
        cols = Aq.first[jj][:, None] + np.arange(4)[None, :]
        msk = np.arange(4)[None, :] < Aq.count[jj][:, None]
        cols = np.where(msk, cols, 0)
        ww = case.w[z][k, cols] * msk
        scale1 = np.sum(np.abs(ww * Aq.vals[jj] * e[z][k, cols]))  # sum |w A e| (reading R20)
        assert abs(t1g[q] - t1) <= 1e-5 * scale1 + 1e-30, (j, t1g[q], t1, scale1)
        assert abs(t2g[q] - t2) <= 1e-5 * t2, (j, t2g[q], t2)
        assert abs(dg[q] - dl) <= 1e-5 * (abs(x32[j]) + abs(dl)) + 1e-7 * MU_W, (j, dg[q], dl)


def test_probe_theta_delta_fixed_state_2d(cfg1):
    cfg, case, g, og, A, codes, amax, Aq = cfg1
    pr = O.Prior(sigma=cfg.sigma, nbhd=8)
    x32, e = _fixed_state(cfg, case, og, Aq, pr)
    with M.Reconstructor(g, M.Prior(sigma=cfg.sigma, neighborhood=8), M.Options(sv_side=cfg.sv_side)) as r:
        r.set_sinogram(case.y, case.w)
        r.set_image(x32.reshape(1, cfg.n, cfg.n))
        vox = np.random.default_rng(0).choice(cfg.n * cfg.n, 300, replace=False)
        vox = np.concatenate([vox, [0, cfg.n - 1, cfg.n * cfg.n - 1]])  # image corners
        t1g, t2g, dg = r.probe(vox)
    _check_probe(og, pr, Aq, case, x32, e, t1g, t2g, dg, vox)


def test_probe_theta_delta_fixed_state_3d_fp32_values():
    cfg = small3d()
    case = make_case(cfg)
    g, og = geoms(cfg)
    A = O.sysmatrix(og)
    pr = O.Prior(sigma=cfg.sigma, nbhd=26)
    x32, e = _fixed_state(cfg, case, og, A, pr, sweeps=2)
    with M.Reconstructor(g, M.Prior(sigma=cfg.sigma, neighborhood=26),
                         M.Options(sv_side=cfg.sv_side, quantize_A=0)) as r:
        r.set_sinogram(case.y, case.w)
        r.set_image(x32.reshape(cfg.nz, cfg.n, cfg.n))
        vox = np.random.default_rng(1).choice(cfg.nz * cfg.n * cfg.n, 200, replace=False)
        t1g, t2g, dg = r.probe(vox)
    _check_probe(og, pr, A, case, x32, e, t1g, t2g, dg, vox)


# ------------------------------------------------------------------ error sinogram (setup)
def test_error_sinogram_equals_y_minus_Ax(cfg1):
    cfg, case, g, og, A, codes, amax, Aq = cfg1
    x = (np.random.default_rng(2).uniform(0, 0.03, cfg.n * cfg.n)).astype(np.float32)
    with M.Reconstructor(g, M.Prior(neighborhood=8), M.Options(sv_side=cfg.sv_side)) as r:
        r.set_sinogram(case.y, case.w)
        r.set_image(x.reshape(1, cfg.n, cfg.n))
        eg = r.error_sinogram()
    eo = O.error_sinogram(og, Aq, case.y.astype(np.float64), x.astype(np.float64))
    np.testing.assert_allclose(eg, eo, atol=2e-6 * np.abs(case.y).max())


# ------------------------------------------------------------------ deterministic tracking
@pytest.mark.parametrize("quant", [1, 0])
def test_deterministic_equit_tracks_sequential_oracle_2d(cfg1, quant):
    """One SV at a time, raster voxel order: the GPU is sequential ICD in a known order, so
    x after each equit must equal the oracle's run over the same order (fp32 tolerance)."""
    cfg, case, g, og, A, codes, amax, Aq = cfg1
    Ause = Aq if quant else A
    pr = O.Prior(sigma=cfg.sigma, nbhd=8)
    order = deterministic_order(cfg.n, 1, cfg.sv_side, 8)
    assert len(order) == cfg.n * cfg.n
    with M.Reconstructor(g, M.Prior(sigma=cfg.sigma, neighborhood=8),
                         M.Options(sv_side=cfg.sv_side, deterministic=1, zero_skip=0, quantize_A=quant)) as r:
        r.set_sinogram(case.y, case.w)
        x = np.zeros(cfg.n * cfg.n)
        e = O.error_sinogram(og, Ause, case.y.astype(np.float64), x)
        for it in range(3):
            st = r.iterate(1)
            assert st["updates"] == cfg.n * cfg.n and st["skipped"] == 0
            O.icd_run(og, pr, Ause, case.w, x, e, 1, zero_skip=False, order=order)
            xg = r.image().ravel()
            err = np.abs(xg - x).max() / np.abs(x).max()
            assert err < 2e-5 * (it + 1), (it, err)
        eg = r.error_sinogram()
    assert np.abs(eg.ravel() - e.ravel()).max() < 1e-4 * np.abs(case.y).max()


def test_deterministic_equit_tracks_sequential_oracle_3d():
    cfg = small3d()
    case = make_case(cfg)
    g, og = geoms(cfg)
    A = O.sysmatrix(og)
    _, _, Aq = O.quantize(A)
    pr = O.Prior(sigma=cfg.sigma, nbhd=26)
    order = deterministic_order(cfg.n, cfg.nz, cfg.sv_side, 26)
    with M.Reconstructor(g, M.Prior(sigma=cfg.sigma, neighborhood=26),
                         M.Options(sv_side=cfg.sv_side, deterministic=1, zero_skip=0)) as r:
        r.set_sinogram(case.y, case.w)
        st = r.iterate(2)
        xg = r.image().ravel()
    x = np.zeros(cfg.nz * cfg.n * cfg.n)
    e = O.error_sinogram(og, Aq, case.y.astype(np.float64), x)
    O.icd_run(og, pr, Aq, case.w, x, e, 2, zero_skip=False, order=order)
    assert st["updates"] == 2 * x.size
    assert np.abs(xg - x).max() / np.abs(x).max() < 5e-5


# ------------------------------------------------------------------ converged parity
@pytest.mark.parametrize("zero_skip,tol_hu,tol_cost", [(0, 1.0, 1e-4), (1, 1.0, 1e-4)])
def test_converged_image_and_cost_match_oracle_cfg1(cfg1, zero_skip, tol_hu, tol_cost):
    """Asynchronous parallel ICD is nondeterministic, but the MAP point is unique: the
    converged GPU image is within 1 HU RMSE of the oracle's and the cost within 1e-4.  With
    zero-skipping and its periodic re-admission (reading R9) the fixed point is still the
    MAP, so the same bound holds against the oracle's no-skip run."""
    cfg, case, g, og, A, codes, amax, Aq = cfg1
    pr = O.Prior(sigma=cfg.sigma, nbhd=8)
    x = np.zeros(cfg.n * cfg.n)
    e = O.error_sinogram(og, Aq, case.y.astype(np.float64), x)
    O.icd_run(og, pr, Aq, case.w, x, e, 150, seed=3000, zero_skip=False)
    with M.Reconstructor(g, M.Prior(sigma=cfg.sigma, neighborhood=8),
                         M.Options(sv_side=cfg.sv_side, zero_skip=zero_skip)) as r:
        r.set_sinogram(case.y, case.w)
        st = r.reconstruct(300)
        xg = r.image().ravel().astype(np.float64)
        eg = r.error_sinogram()
    assert st["equits"] >= 300
    rm = O.rmse_hu(xg, x)
    assert rm < tol_hu, rm
    cg = O.cost(og, pr, Aq, case.y, case.w, xg)
    co = O.cost(og, pr, Aq, case.y, case.w, x)
    assert abs(cg - co) <= tol_cost * abs(co), (cg, co)
    # e stays consistent with y - A x (fp32 drift bound)
    eo = O.error_sinogram(og, Aq, case.y.astype(np.float64), xg)
    assert np.abs(eg.ravel() - eo.ravel()).max() < 1e-3 * np.abs(case.y).max()


@pytest.mark.parametrize("zero_skip,tol_hu,tol_cost", [(0, 1.0, 1e-4), (1, 1.0, 1e-4)])
def test_converged_3d_matches_oracle(zero_skip, tol_hu, tol_cost):
    """The MAP point is unique: 1 HU / 1e-4 (BASELINE.json) against the oracle's no-skip run,
    with or without zero-skipping, whose periodic re-admission (reading R9) keeps the
    MAP as the fixed point."""
    cfg = small3d()
    case = make_case(cfg)
    g, og = geoms(cfg)
    A = O.sysmatrix(og)
    _, _, Aq = O.quantize(A)
    pr = O.Prior(sigma=cfg.sigma, nbhd=26)
    x = np.zeros(cfg.nz * cfg.n * cfg.n)
    e = O.error_sinogram(og, Aq, case.y.astype(np.float64), x)
    O.icd_run(og, pr, Aq, case.w, x, e, 120, seed=3000, zero_skip=False)
    with M.Reconstructor(g, M.Prior(sigma=cfg.sigma, neighborhood=26),
                         M.Options(sv_side=cfg.sv_side, zero_skip=zero_skip)) as r:
        r.set_sinogram(case.y, case.w)
        r.reconstruct(240)
        xg = r.image().ravel().astype(np.float64)
    assert O.rmse_hu(xg, x) < tol_hu
    cg = O.cost(og, pr, Aq, case.y, case.w, xg)
    co = O.cost(og, pr, Aq, case.y, case.w, x)
    assert abs(cg - co) <= tol_cost * abs(co)


SWEEP_SMALL = [  # (phantom, baggage seed, lambda0, views, SV side): BASELINE configs[4]'s axes at N = 64
    ("shepp_logan", 0, 1e3, 180, 5),
    ("baggage", 0, 1e4, 90, 7),
    ("baggage", 1, 1e5, 360, 9),
    ("shepp_logan", 0, 1e5, 90, 9),
]


@pytest.mark.parametrize("case", SWEEP_SMALL, ids=[f"{c[0]}{c[1]}-l{int(c[2])}-v{c[3]}-s{c[4]}" for c in SWEEP_SMALL])
def test_sweep_cases_converge_to_oracle(case):
    """The sweep's variety (BASELINE.json configs[4]: phantom incl. baggage-like scenes with a
    large air fraction, dose, view count, SV side; M = 2N as in the paper) at a size the oracle
    converges in seconds: converged image within 1 HU and cost within 1e-4 of the oracle's."""
    ph, bseed, lam, v, side = case
    cfg = WorkloadConfig("sweep-small", 64, 1, v, 128, side, 8, 0.002, phantom=ph, lambda0=lam)
    c = make_case(cfg, 100 + bseed)
    g, og = geoms(cfg)
    A = O.sysmatrix(og)
    _, _, Aq = O.quantize(A)
    pr = O.Prior(sigma=cfg.sigma, nbhd=8)
    x = np.zeros(cfg.n * cfg.n)
    e = O.error_sinogram(og, Aq, c.y.astype(np.float64), x)
    O.icd_run(og, pr, Aq, c.w, x, e, 150, seed=3000, zero_skip=False)
    with M.Reconstructor(g, M.Prior(sigma=cfg.sigma, neighborhood=8),
                         M.Options(sv_side=side, zero_skip=0)) as r:
        r.set_sinogram(c.y, c.w)
        r.reconstruct(300)
        xg = r.image().ravel().astype(np.float64)
    assert O.rmse_hu(xg, x) < 1.0, O.rmse_hu(xg, x)
    cg = O.cost(og, pr, Aq, c.y, c.w, xg)
    co = O.cost(og, pr, Aq, c.y, c.w, x)
    assert abs(cg - co) <= 1e-4 * abs(co), (cg, co)


# ------------------------------------------------------------------ scheduler + accounting
def test_iteration_accounting_and_selection_fractions(cfg1):
    """Alg3:17-22: iteration 1 visits every SV of every slice; later iterations
    ceil(25 %) per slice (no threshold when batch_svs = 0); equits = updates / N."""
    cfg = small3d()
    case = make_case(cfg)
    g, _ = geoms(cfg)
    with M.Reconstructor(g, M.Prior(sigma=cfg.sigma, neighborhood=26),
                         M.Options(sv_side=cfg.sv_side, zero_skip=0)) as r:
        r.set_sinogram(case.y, case.w)
        nsv = r.sizes()["nsv"]
        st1 = r.iterate(1)
        assert st1["sv_visits"] == nsv * cfg.nz
        assert st1["updates"] == cfg.nz * cfg.n * cfg.n
        assert st1["equits"] == pytest.approx(1.0)
        for _ in range(4):
            st = r.iterate(1)
            assert st["sv_visits"] == int(np.ceil(0.25 * nsv)) * cfg.nz
            assert st["skipped"] == 0


def test_batch_threshold_drops_small_remainders(cfg1):
    """Alg3:26-27 / P:225: with BATCH_SIZE = B, a colour group's remainder smaller than B/4 is
    not launched.  cfg1 (8x8 SVs, 16 per colour): B = 12 -> remainder 4 >= 3 kept in iteration 1;
    B = 10, threshold 8 -> remainder 6 dropped from every colour."""
    cfg, case, g, *_ = cfg1
    with M.Reconstructor(g, M.Prior(sigma=cfg.sigma, neighborhood=8),
                         M.Options(sv_side=cfg.sv_side, zero_skip=0, batch_svs=12)) as r:
        r.set_sinogram(case.y, case.w)
        assert r.iterate(1)["sv_visits"] == 64
    with M.Reconstructor(g, M.Prior(sigma=cfg.sigma, neighborhood=8),
                         M.Options(sv_side=cfg.sv_side, zero_skip=0, batch_svs=10, batch_threshold=8)) as r:
        r.set_sinogram(case.y, case.w)
        assert r.iterate(1)["sv_visits"] == 4 * 10


def test_zero_skip_counts(cfg1):
    """with zero-skipping, an all-zero sinogram leaves x = 0 and, from iteration 2 on,
    every voxel is skipped."""
    cfg, case, g, *_ = cfg1
    z = np.zeros_like(case.y)
    with M.Reconstructor(g, M.Prior(sigma=cfg.sigma, neighborhood=8), M.Options(sv_side=cfg.sv_side)) as r:
        r.set_sinogram(z, case.w)
        st = r.iterate(1)
        assert st["updates"] == cfg.n * cfg.n
        st = r.iterate(1)
        assert st["updates"] == 0 and st["skipped"] > 0
        assert np.all(r.image() == 0)


# ------------------------------------------------------------------ boundary errors
def test_invalid_arguments_rejected():
    cfg = CONFIGS["cfg1"]
    g, _ = geoms(cfg)
    for pr in (M.Prior(q=1.5), M.Prior(p=0.5), M.Prior(sigma=0.0), M.Prior(neighborhood=6)):
        with pytest.raises(M.MbirError) as ei:
            M.Reconstructor(g, pr)
        assert ei.value.code == -1
    with pytest.raises(M.MbirError):
        M.Reconstructor(M.Geometry(64, 64, 1, 4.0, 90, 96, 0.5))  # K > 4 channels per view
    with M.Reconstructor(g, M.Prior(neighborhood=8)) as r:
        with pytest.raises(M.MbirError) as ei:
            r.reconstruct(1.0)
        assert ei.value.code == -4  # ESTATE: no sinogram
        y = np.zeros((1, cfg.nviews, cfg.nchannels), np.float32)
        w = -np.ones_like(y)
        with pytest.raises(M.MbirError) as ei:
            r.set_sinogram(y, w)
        assert ei.value.code == -1
        y[0, 0, 0] = np.nan
        with pytest.raises(M.MbirError):
            r.set_sinogram(y, np.ones_like(y))


# ------------------------------------------------------------------ the bench's launch shape
def mini720():
    """The bench's kernel shape on an image the oracle handles: 720 views (4 views per lane, six
    128-view warps), channel pitch dxy/2 as in the paper geometry (K = 4, 2.4K nnz per voxel),
    SV side 9 with a ragged last SV column/row, two slices, 26-neighbourhood."""
    return WorkloadConfig("mini720", 48, 2, 720, 96, 9, 26, 0.005)


@pytest.fixture(scope="module")
def m720():
    cfg = mini720()
    case = make_case(cfg)
    g, og = geoms(cfg)
    A = O.sysmatrix(og)
    _, _, Aq = O.quantize(A)
    return cfg, case, g, og, Aq


@pytest.mark.parametrize("cluster", [1, 2])
def test_bench_shape_deterministic_tracks_oracle(m720, cluster):
    """The launch configuration bench.py times (uint8 A, 4 views per lane, 6 view warps + the
    delta and prior warps, one CTA per task): deterministic order, 2 equits, against the
    sequential oracle."""
    cfg, case, g, og, Aq = m720
    pr = O.Prior(sigma=cfg.sigma, nbhd=26)
    order = deterministic_order(cfg.n, cfg.nz, cfg.sv_side, 26)
    with M.Reconstructor(g, M.Prior(sigma=cfg.sigma, neighborhood=26),
                         M.Options(sv_side=cfg.sv_side, deterministic=1, zero_skip=0, cluster=cluster)) as r:
        assert r.sizes()["cluster"] == cluster
        r.set_sinogram(case.y, case.w)
        x = np.zeros(cfg.nz * cfg.n * cfg.n)
        e = O.error_sinogram(og, Aq, case.y.astype(np.float64), x)
        for it in range(2):
            st = r.iterate(1)
            assert st["updates"] == x.size and st["skipped"] == 0
            O.icd_run(og, pr, Aq, case.w, x, e, 1, zero_skip=False, order=order)
            xg = r.image().ravel()
            err = np.abs(xg - x).max() / np.abs(x).max()
            assert err < 3e-5 * (it + 1), (it, err)
        eg = r.error_sinogram()
    assert np.abs(eg.ravel() - e.ravel()).max() < 1e-4 * np.abs(case.y).max()


@pytest.mark.parametrize("cluster,vps", [(1, 1), (2, 1), (1, 2)])
def test_bench_shape_converged_matches_oracle(m720, cluster, vps):
    """Asynchronous GPU-ICD in the bench's launch shape (persistent grid, random orders, 25 %
    SV selection, zero-skipping off) reaches the oracle's MAP point: 1 HU / 1e-4 -- also with a
    2-CTA cluster per task and with voxel pairs (same fixed points: a pair's update of x and e is
    the sum of two exact single-voxel updates from one state)."""
    cfg, case, g, og, Aq = m720
    pr = O.Prior(sigma=cfg.sigma, nbhd=26)
    x = np.zeros(cfg.nz * cfg.n * cfg.n)
    e = O.error_sinogram(og, Aq, case.y.astype(np.float64), x)
    O.icd_run(og, pr, Aq, case.w, x, e, 80, seed=3000, zero_skip=False)
    with M.Reconstructor(g, M.Prior(sigma=cfg.sigma, neighborhood=26),
                         M.Options(sv_side=cfg.sv_side, zero_skip=0, cluster=cluster, voxels_per_step=vps)) as r:
        assert r.sizes()["voxels_per_step"] == vps
        r.set_sinogram(case.y, case.w)
        r.reconstruct(200)
        xg = r.image().ravel().astype(np.float64)
    assert O.rmse_hu(xg, x) < 1.0
    cg = O.cost(og, pr, Aq, case.y, case.w, xg)
    co = O.cost(og, pr, Aq, case.y, case.w, x)
    assert abs(cg - co) <= 1e-4 * abs(co), (cg, co)


def test_cluster_option_validation():
    """CTAs per SV task (include/mbir.h mbir_options.cluster): 0 (auto) and 1 = one CTA; 2 = a
    2-CTA cluster splitting the views, which needs > 128 views in an even number of 128-view warps;
    anything else is EINVAL."""
    cfg = CONFIGS["cfg1"]  # 90 views: three warps of 1 view per lane
    g, _ = geoms(cfg)
    for bad in (2, 3, -1):
        with pytest.raises(M.MbirError) as ei:
            M.Reconstructor(g, M.Prior(neighborhood=8), M.Options(sv_side=cfg.sv_side, cluster=bad))
        assert ei.value.code == -1
    with M.Reconstructor(g, M.Prior(neighborhood=8), M.Options(sv_side=cfg.sv_side)) as r:
        assert r.sizes()["cluster"] == 1
        assert r.sizes()["threads_per_cta"] == 32 * (3 + 2)
    cfg = mini720()
    g, _ = geoms(cfg)
    with M.Reconstructor(g, M.Prior(neighborhood=26), M.Options(sv_side=cfg.sv_side, cluster=2)) as r:
        assert r.sizes()["cluster"] == 2 and r.sizes()["threads_per_cta"] == 32 * (3 + 2)


def test_large_svs_use_two_windows_and_a_cluster():
    """NEXT-2 (larger SVs): at the paper's pitch (dc = dxy/2) side 9 needs <= 29
    band rows (one 32-float window per row, one CTA); sides 11 and 13 need 35-41 rows: two
    windows per row, and auto cluster selection splits the SV buffer over a 2-CTA cluster; a side
    whose band exceeds 61 rows is EINVAL."""
    for side, want_cl in ((9, 1), (11, 2), (13, 2)):
        cfg = WorkloadConfig("mini720", 48, 2, 720, 96, side, 26, 0.005)
        g, _ = geoms(cfg)
        with M.Reconstructor(g, M.Prior(neighborhood=26), M.Options(sv_side=side)) as r:
            s = r.sizes()
            assert s["cluster"] == want_cl, (side, s)
            assert (s["svb_rows"] > 29) == (side > 9), (side, s)
    cfg = WorkloadConfig("big", 96, 1, 720, 192, 24, 8, 0.005)
    g, _ = geoms(cfg)
    with pytest.raises(M.MbirError) as ei:
        M.Reconstructor(g, M.Prior(neighborhood=8), M.Options(sv_side=24))
    assert ei.value.code == -1


@pytest.mark.parametrize("side", [11, 13])
def test_large_sv_converged_matches_oracle(m720, side):
    """Asynchronous GPU-ICD with side-11 / side-13 SVs (two-window bands, 2-CTA clusters) reaches
    the oracle's MAP point on the bench-shaped case: 1 HU / 1e-4."""
    cfg, case, g, og, Aq = m720
    pr = O.Prior(sigma=cfg.sigma, nbhd=26)
    x = np.zeros(cfg.nz * cfg.n * cfg.n)
    e = O.error_sinogram(og, Aq, case.y.astype(np.float64), x)
    O.icd_run(og, pr, Aq, case.w, x, e, 80, seed=3000, zero_skip=False)
    with M.Reconstructor(g, M.Prior(sigma=cfg.sigma, neighborhood=26), M.Options(sv_side=side, zero_skip=0)) as r:
        assert r.sizes()["cluster"] == 2
        r.set_sinogram(case.y, case.w)
        r.reconstruct(200)
        xg = r.image().ravel().astype(np.float64)
    assert O.rmse_hu(xg, x) < 1.0
    cg = O.cost(og, pr, Aq, case.y, case.w, xg)
    co = O.cost(og, pr, Aq, case.y, case.w, x)
    assert abs(cg - co) <= 1e-4 * abs(co), (cg, co)


def test_large_sv_odd_view_warps_padded_cluster_matches_oracle():
    """360 views at the paper's pitch with side-13 SVs: the SV buffer (41 rows) exceeds one CTA and
    the 3 view warps cannot be split evenly over a 2-CTA cluster, so the library pads a fourth,
    empty view warp (views >= 360 carry zero records) and clusters.  Converged image and cost
    match the oracle's MAP (1 HU / 1e-4); the padded run of side 9 (one CTA, odd warps) and an
    explicit cluster = 2 with 360 views are accepted too."""
    cfg = WorkloadConfig("mini360", 48, 2, 360, 96, 13, 26, 0.005)
    case = make_case(cfg)
    g, og = geoms(cfg)
    _, _, Aq = O.quantize(O.sysmatrix(og))
    pr = O.Prior(sigma=cfg.sigma, nbhd=26)
    x = np.zeros(cfg.nz * cfg.n * cfg.n)
    e = O.error_sinogram(og, Aq, case.y.astype(np.float64), x)
    O.icd_run(og, pr, Aq, case.w, x, e, 80, seed=3000, zero_skip=False)
    with M.Reconstructor(g, M.Prior(sigma=cfg.sigma, neighborhood=26), M.Options(sv_side=13)) as r:
        s = r.sizes()
        assert s["cluster"] == 2 and s["threads_per_cta"] == 32 * (2 + 2), s
        r.set_sinogram(case.y, case.w)
        r.reconstruct(200)
        xg = r.image().ravel().astype(np.float64)
    assert O.rmse_hu(xg, x) < 1.0
    cg = O.cost(og, pr, Aq, case.y, case.w, xg)
    co = O.cost(og, pr, Aq, case.y, case.w, x)
    assert abs(cg - co) <= 1e-4 * abs(co), (cg, co)
    with M.Reconstructor(g, M.Prior(neighborhood=26), M.Options(sv_side=9)) as r:
        assert r.sizes()["cluster"] == 1 and r.sizes()["threads_per_cta"] == 32 * (3 + 2)
    with M.Reconstructor(g, M.Prior(neighborhood=26), M.Options(sv_side=9, cluster=2)) as r:
        assert r.sizes()["cluster"] == 2 and r.sizes()["threads_per_cta"] == 32 * (2 + 2)


def test_voxels_per_step_option_validation():
    """mbir_options.voxels_per_step: 0 (auto) = 1, 1, or 2 (voxel pairs, uint8 A and one CTA per
    task only); anything else is EINVAL."""
    cfg = mini720()
    g, _ = geoms(cfg)
    for kw in ({"voxels_per_step": 3}, {"voxels_per_step": -1}, {"voxels_per_step": 2, "quantize_A": 0},
               {"voxels_per_step": 2, "cluster": 2}):
        with pytest.raises(M.MbirError) as ei:
            M.Reconstructor(g, M.Prior(neighborhood=26), M.Options(sv_side=cfg.sv_side, **kw))
        assert ei.value.code == -1, kw
    for v, want in ((0, 1), (1, 1), (2, 2)):
        with M.Reconstructor(g, M.Prior(neighborhood=26), M.Options(sv_side=cfg.sv_side, voxels_per_step=v)) as r:
            assert r.sizes()["voxels_per_step"] == want


# ------------------------------------------------------------------ FBP initial image (R23)
def test_fbp_init_matches_reference_and_converges(cfg1):
    """mbir_init_fbp: the device FBP equals the float64 textbook reference (oracle.fbp) to fp32
    accuracy, e is reset to y - A x, and ICD from it reaches the same MAP point as the oracle."""
    cfg, case, g, og, A, codes, amax, Aq = cfg1
    ref = O.fbp(og, case.y)
    with M.Reconstructor(g, M.Prior(sigma=cfg.sigma, neighborhood=8),
                         M.Options(sv_side=cfg.sv_side, zero_skip=0)) as r:
        r.set_sinogram(case.y, case.w)
        r.init_fbp()
        x0 = r.image().astype(np.float64)
        e0 = r.error_sinogram()
        assert np.abs(x0 - ref).max() <= 2e-5 * np.abs(ref).max(), np.abs(x0 - ref).max()
        eo = O.error_sinogram(og, Aq, case.y.astype(np.float64), x0.ravel())
        assert np.abs(e0.ravel() - eo.ravel()).max() < 1e-4 * np.abs(case.y).max()
        r.reconstruct(300)
        xg = r.image().ravel().astype(np.float64)
    pr = O.Prior(sigma=cfg.sigma, nbhd=8)
    x = np.zeros(cfg.n * cfg.n)
    e = O.error_sinogram(og, Aq, case.y.astype(np.float64), x)
    O.icd_run(og, pr, Aq, case.w, x, e, 150, seed=3000, zero_skip=False)
    assert O.rmse_hu(xg, x) < 1.0
    cg = O.cost(og, pr, Aq, case.y, case.w, xg)
    co = O.cost(og, pr, Aq, case.y, case.w, x)
    assert abs(cg - co) <= 1e-4 * abs(co)


def test_fbp_init_3d_slab_and_state_errors():
    cfg = small3d()
    case = make_case(cfg)
    g, og = geoms(cfg)
    ref = O.fbp(og, case.y)
    with M.Reconstructor(g, M.Prior(sigma=cfg.sigma, neighborhood=26), M.Options(sv_side=cfg.sv_side)) as r:
        with pytest.raises(M.MbirError):
            r.init_fbp()  # no sinogram yet: MBIR_ESTATE
        r.set_sinogram(case.y, case.w)
        r.init_fbp()
        x0 = r.image().astype(np.float64)
    assert np.abs(x0 - ref).max() <= 2e-5 * np.abs(ref).max()


def test_2d_slice_with_many_svs_does_not_collapse():
    """One 2-D slice with 676 SVs (169 per colour): with all of a colour's SVs in flight at once
    the first sweeps from x0 = 0 overshoot, clip whole SVs to 0 and zero-skip freezes them
    (the image stalls at x = 0).  batch_svs = 0 (auto) caps concurrent SVs per slice (reading
    R22); the GPU then converges to the oracle's fixed point like any other case."""
    cfg = WorkloadConfig("sweep-128", 128, 1, 90, 256, 5, 8, 0.003, lambda0=1e3)
    c = make_case(cfg, 100)
    g, og = geoms(cfg)
    _, _, Aq = O.quantize(O.sysmatrix(og))
    pr = O.Prior(sigma=cfg.sigma, nbhd=8)
    x = np.zeros(cfg.n * cfg.n)
    e = O.error_sinogram(og, Aq, c.y.astype(np.float64), x)
    O.icd_run(og, pr, Aq, c.w, x, e, 120, seed=3000, zero_skip=False)
    with M.Reconstructor(g, M.Prior(sigma=cfg.sigma, neighborhood=8), M.Options(sv_side=5)) as r:
        r.set_sinogram(c.y, c.w)
        r.reconstruct(160)
        xg = r.image().ravel().astype(np.float64)
    assert xg.max() > 0.5 * x.max()
    # zero-skip with re-admission (reading R9) reaches the no-skip MAP
    assert O.rmse_hu(xg, x) < 1.0, O.rmse_hu(xg, x)


def test_zero_skip_prefilter_path_matches_oracle():
    """Iterations >= 2 without batching flag fully zero-skipped SV visits per phase and account
    them at task fetch (api.cu / sched.cu k_zero_flags).  A whole-group batch on a 3-D baggage case
    (large air fraction) exercises it: empty visits are reported, the accounting stays consistent
    and the converged image matches the oracle's MAP (1 HU / 1e-4)."""
    cfg = WorkloadConfig("mini3d-bag", 40, 4, 60, 64, 7, 26, 0.002, phantom="baggage")
    case = make_case(cfg, 101)
    g, og = geoms(cfg)
    _, _, Aq = O.quantize(O.sysmatrix(og))
    pr = O.Prior(sigma=cfg.sigma, nbhd=26)
    x = np.zeros(cfg.nz * cfg.n * cfg.n)
    e = O.error_sinogram(og, Aq, case.y.astype(np.float64), x)
    O.icd_run(og, pr, Aq, case.w, x, e, 120, seed=3000, zero_skip=False)
    nvox = cfg.nz * cfg.n * cfg.n
    with M.Reconstructor(g, M.Prior(sigma=cfg.sigma, neighborhood=26),
                         M.Options(sv_side=cfg.sv_side, batch_svs=1000, batch_threshold=0)) as r:
        r.set_sinogram(case.y, case.w)
        st1 = r.iterate(1)
        assert st1["updates"] == nvox and st1["sv_visits_empty"] == 0  # no skipping in iteration 1
        empty = 0
        for _ in range(30):
            st = r.iterate(1)
            assert st["sv_visits_empty"] <= st["sv_visits"]
            empty += st["sv_visits_empty"]
        assert empty > 0
        r.reconstruct(200)
        xg = r.image().ravel().astype(np.float64)
    # the pre-filtered zero-skip path with re-admission (reading R9) reaches the no-skip MAP
    assert O.rmse_hu(xg, x) < 1.0, O.rmse_hu(xg, x)
    cg = O.cost(og, pr, Aq, case.y, case.w, xg)
    co = O.cost(og, pr, Aq, case.y, case.w, x)
    assert abs(cg - co) <= 1e-4 * abs(co)


@pytest.mark.parametrize("name", ["cfg3", "cfg4"])
def test_paper_scale_error_sinogram_consistent_on_sampled_rays(name):
    """Configs 3 and 4 at full size (512^2 x 1 / x 64, 720 views x 1024 channels, side 9) after
    asynchronous iterations in the bench's kernel configuration: the error sinogram the update
    kernel maintains (SVB scatter + atomic write-back, a6/a7) equals y - A x for the GPU's own x on
    sampled (slice, view, channel) entries, each recomputed by the oracle from the columns of every
    voxel on that ray (the full A is too large for the oracle)."""
    import torch
    from synth import make_sinogram_torch
    cfg = CONFIGS[name]
    g, og = geoms(cfg, nz=1)
    g = M.Geometry(cfg.n, cfg.n, cfg.nz, cfg.dxy, cfg.nviews, cfg.nchannels, cfg.dchannel)
    y, w = make_sinogram_torch(cfg, 0, "cuda")
    with M.Reconstructor(g, M.Prior(sigma=cfg.sigma, neighborhood=cfg.nbhd), M.Options(sv_side=cfg.sv_side)) as r:
        r.set_sinogram(y, w)
        r.iterate(3)
        xs = r.image().astype(np.float64)
        eg = r.error_sinogram()
    ys = y.cpu().numpy()
    assert np.isfinite(xs).all() and xs.min() >= 0 and xs.max() > 0
    rng = np.random.default_rng(11)
    n, dxy, dc = cfg.n, cfg.dxy, cfg.dchannel
    c = (np.arange(n) - 0.5 * (n - 1)) * dxy
    X, Y = np.meshgrid(c, c)  # [iy][ix]
    t0 = -0.5 * cfg.nchannels * dc
    busy = 0
    cols = {}
    for _ in range(6):
        z = int(rng.integers(cfg.nz))
        k = int(rng.integers(cfg.nviews))
        m = int(rng.integers(cfg.nchannels // 4, 3 * cfg.nchannels // 4))
        x = xs[z]
        th = k * np.pi / cfg.nviews
        h = 0.5 * dxy * (abs(np.cos(th)) + abs(np.sin(th)))
        tm = t0 + (m + 0.5) * dc
        iy, ix = np.nonzero((np.abs(X * np.cos(th) + Y * np.sin(th) - tm) < h + dc) & (x > 0))
        acc = 0.0
        for yy, xx in zip(iy, ix):
            key = (int(xx), int(yy))
            if key not in cols:
                f, cnt, v, _ = O.sysmatrix_column(og, key[0], key[1], K=4)
                codes, amax = O.quantize_column(v, cnt)
                cols[key] = (f, cnt, codes, float(np.float32(amax / 255.0)))
            f, cnt, codes, sc = cols[key]
            if cnt[k] == 0 or not (f[k] <= m < f[k] + cnt[k]):
                continue
            acc += float(codes[k, m - f[k]]) * sc * x[yy, xx]
        ref = float(ys[z, k, m]) - acc
        busy += acc > 0.1 * abs(float(ys[z, k, m]))
        assert abs(float(eg[z, k, m]) - ref) <= 2e-4 * max(1.0, abs(float(ys[z, k, m]))), (z, k, m, eg[z, k, m], ref)
    assert busy >= 3  # the sampled rays cross the reconstructed object


def test_bench_template_mid_size_3d_converges_to_oracle_map():
    """The bench's kernel template at a size the oracle can converge: 96^2 x 8
    slices, 720 views x 192 channels (dc = dxy/2, paper pitch ratio), SV side 9, uint8 A,
    26-neighbourhood, zero-skip with re-admission, whole colour groups per launch (unbatched, as
    cfg4 runs), from x0 = 0 -- against the oracle's no-skip MAP (slice-parity threads): 1 HU / 1e-4."""
    cfg = WorkloadConfig("mid3d", 96, 8, 720, 192, 9, 26, 0.005)
    case = make_case(cfg)
    g, og = geoms(cfg)
    _, _, Aq = O.quantize(O.sysmatrix(og))
    pr = O.Prior(sigma=cfg.sigma, nbhd=26)
    x = O.fbp(og, case.y).ravel().copy()
    e = O.error_sinogram(og, Aq, case.y.astype(np.float64), x)
    O.icd_run_zpar(og, pr, Aq, case.w, x, e, 60, seed=3000, zero_skip=False)
    with M.Reconstructor(g, M.Prior(sigma=cfg.sigma, neighborhood=26),
                         M.Options(sv_side=cfg.sv_side, batch_svs=100000, batch_threshold=0)) as r:
        r.set_sinogram(case.y, case.w)
        r.reconstruct(120)
        xg = r.image().ravel().astype(np.float64)
    assert O.rmse_hu(xg, x) < 1.0, O.rmse_hu(xg, x)
    cg = O.cost(og, pr, Aq, case.y, case.w, xg)
    co = O.cost(og, pr, Aq, case.y, case.w, x)
    assert abs(cg - co) <= 1e-4 * abs(co), (cg, co)
