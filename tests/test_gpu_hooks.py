"""GPU parity of the hot kernel's own arithmetic and of the device-side bookkeeping, through the
C-ABI test hooks (VERDICT r1 "What's weak" 1-2):

  - every update k_svicd executes (theta1, theta2, delta of Alg. 1, as its delta chain
    used them) against the oracle's orc_voxel_update at the same state (reading R20's 1e-5),
    in deterministic mode, replayed update by update;
  - the device RMSE-HU reduction against oracle.rmse_hu;
  - the scheduler's top-25 % / random-25 % selections and the checkerboard colouring (Alg3:17-23,
    P:203-225, reading R14) against numpy on the exported update amounts.
"""
import numpy as np
import pytest

import oracle as O
import paper_conf_ppopp_sabnewkbrm17_b200 as M
from synth import CONFIGS, WorkloadConfig, make_case
from tests.helpers import deterministic_order, geoms

pytestmark = pytest.mark.gpu

MU_W = 0.02


def _state(cfg, case, og, Aq, nbhd, sweeps):
    """A non-trivial fixed state: the oracle's x after `sweeps` random-order sweeps (float32),
    and e = y - A x for it."""
    pr = O.Prior(sigma=cfg.sigma, nbhd=nbhd)
    x = np.zeros(og.nx * og.ny * og.nz)
    e = O.error_sinogram(og, Aq, case.y.astype(np.float64), x)
    O.icd_run(og, pr, Aq, case.w, x, e, sweeps, seed=5, zero_skip=False)
    return pr, x.astype(np.float32)


def _replay(og, pr, Aq, case, x32, vox, t1g, t2g, dg):
    """Walk the GPU's update record: at each step the oracle computes Alg. 1 for that voxel at
    the current state, which is then advanced with the GPU's own delta (so every comparison is
    a fixed-state comparison and fp32 drift of the state does not accumulate into it).  A record
    flagged DUMP_SAME_STATE (the second voxel of a pair) is computed at the state before the
    previous record's update: the pair's updates are applied together after both checks."""
    plane = og.nx * og.ny
    V = og.nviews
    x = x32.astype(np.float64).copy()
    e = O.error_sinogram(og, Aq, case.y.astype(np.float64), x)
    w = case.w.astype(np.float64)
    k = np.arange(V)[:, None]
    worst = np.zeros(3)
    same = (vox & M.DUMP_SAME_STATE) != 0
    vox = vox & (M.DUMP_SAME_STATE - 1)
    pending = []  # (j, z, cols, msk, a, delta) of the updates computed from the current state
    for q in range(len(vox)):
        if not same[q]:
            for j, z, cols, msk, a, d in pending:  # advance with the GPU's updates (Alg1:8-11)
                x[j] += d
                np.subtract.at(e[z], (np.broadcast_to(k, cols.shape)[msk], cols[msk]), a[msk] * d)
            pending = []
        j = int(vox[q])
        jj, z = j % plane, j // plane
        t1, t2, dl = O.voxel_update(og, pr, Aq, case.w, x, e, j, apply=False)
        cols = Aq.first[jj][:, None] + np.arange(4)[None, :]
        msk = np.arange(4)[None, :] < Aq.count[jj][:, None]
        cols = np.where(msk, cols, 0)
        a = Aq.vals[jj] * msk
        s1 = np.sum(np.abs(w[z][k, cols] * a * e[z][k, cols]))  # sum |w A e| (reading R20)
        # reading R20: delta within 1e-5 of (|x_j| + |delta|) plus the change a theta1 error within
        # its own bound (1e-5 sum|wAe|) can cause: |d delta / d theta1| = 1/(theta2 + 2 sum b~)
        # <= 1/theta2, which matters where sum w A e cancels (theta1 << sum|wAe|)
        dtol = 1e-5 * (abs(x[j]) + abs(dl) + s1 / t2) + 1e-7 * MU_W
        r = (abs(t1g[q] - t1) / (s1 + 1e-30), abs(t2g[q] - t2) / t2, abs(dg[q] - dl) / dtol)
        worst = np.maximum(worst, r)
        assert r[0] <= 1e-5, (q, j, t1g[q], t1, s1)
        assert r[1] <= 1e-5, (q, j, t2g[q], t2)
        assert r[2] <= 1.0, (q, j, dg[q], dl, x[j], s1 / t2)
        pending.append((j, z, cols, msk, a, float(dg[q])))
    return worst


CASES = {
    # (config, nbhd, quantize_A, sweeps of the oracle to reach the fixed state, CTAs per task,
    #  voxels per step)
    "cfg1-u8": (CONFIGS["cfg1"], 8, 1, 3, 1, 1),
    "cfg1-f32": (CONFIGS["cfg1"], 8, 0, 3, 1, 1),
    "mini720-u8": (WorkloadConfig("mini720", 48, 2, 720, 96, 9, 26, 0.005), 26, 1, 2, 1, 1),
    "mini720-u8-cluster2": (WorkloadConfig("mini720", 48, 2, 720, 96, 9, 26, 0.005), 26, 1, 2, 2, 1),
    "mini3d-f32": (WorkloadConfig("mini3d", 40, 4, 60, 64, 7, 26, 0.002), 26, 0, 2, 1, 1),
    "cfg1-u8-pairs": (CONFIGS["cfg1"], 8, 1, 3, 1, 2),
    "mini720-u8-pairs": (WorkloadConfig("mini720", 48, 2, 720, 96, 9, 26, 0.005), 26, 1, 2, 1, 2),
    "mini3d-u8-pairs-odd": (WorkloadConfig("mini3d", 40, 4, 60, 64, 7, 26, 0.002), 26, 1, 2, 1, 2),
    # side 11 at the paper's pitch: 35-row bands (two 32-float windows per band row in the pack and
    # write-back), the SV buffer held by a 2-CTA cluster (NEXT-2)
    "mini720-u8-side11-cluster2": (WorkloadConfig("mini720", 48, 2, 720, 96, 11, 26, 0.005), 26, 1, 2, 2, 1),
}


@pytest.mark.parametrize("name", list(CASES))
def test_hot_kernel_every_update_matches_oracle(name):
    """The fused update kernel's own theta1, theta2 (reduced by the kernel in this first iteration
    after set_sinogram) and delta (neighbour-corrected prior) for every update of one deterministic
    sweep from a non-trivial state, against Alg. 1 in the oracle at the identical state: reading
    R20's 1e-5.  mini720 is the bench's launch shape (720 views, 4 views per lane, six view warps,
    uint8 A, 26-neighbourhood); cluster2 splits every task's views over a 2-CTA cluster that
    exchanges the partial sums through distributed shared memory; *-pairs run the voxel-pair
    kernel (two voxels per step from one state), replayed pair by pair; mini3d's
    side-7 tiles of a 40-pixel slice leave odd visits (a lone last voxel)."""
    cfg, nbhd, quant, sweeps, cl, kv = CASES[name]
    case = make_case(cfg)
    g, og = geoms(cfg)
    A = O.sysmatrix(og)
    Ause = O.quantize(A)[2] if quant else A
    pr, x32 = _state(cfg, case, og, Ause, nbhd, sweeps)
    nvox = x32.size
    with M.Reconstructor(g, M.Prior(sigma=cfg.sigma, neighborhood=nbhd),
                         M.Options(sv_side=cfg.sv_side, deterministic=1, zero_skip=0, quantize_A=quant,
                                   cluster=cl, voxels_per_step=kv)) as r:
        assert r.sizes()["cluster"] == cl and r.sizes()["voxels_per_step"] == kv
        r.set_sinogram(case.y, case.w)
        r.set_image(x32.reshape(cfg.nz, cfg.n, cfg.n))
        r.set_update_dump(nvox + 16)
        st = r.iterate(1)
        vox, t1g, t2g, dg, n = r.update_dump(nvox + 16)
    assert st["updates"] == nvox and n == nvox
    same = (vox & M.DUMP_SAME_STATE) != 0
    order = deterministic_order(cfg.n, cfg.nz, cfg.sv_side, nbhd)
    np.testing.assert_array_equal(vox & (M.DUMP_SAME_STATE - 1), order)
    # pairs within each SV visit (runs of one (slice, SV) in the order): positions 1, 3, 5, ...
    # of a visit share the state of the update before them
    s = cfg.sv_side
    iz, iy, ix = order // (cfg.n * cfg.n), (order // cfg.n) % cfg.n, order % cfg.n
    visit = iz * 10 ** 6 + (iy // s) * 1000 + ix // s
    pos = np.zeros(len(order), np.int64)
    for q in range(1, len(order)):
        pos[q] = pos[q - 1] + 1 if visit[q] == visit[q - 1] else 0
    np.testing.assert_array_equal(same, (pos % 2 == 1) if kv == 2 else np.zeros_like(same))
    worst = _replay(og, pr, Ause, case, x32, vox, t1g, t2g, dg)
    print(name, "worst error / tolerance  theta1 %.3g  theta2 %.3g  delta %.3g" % (worst[0] / 1e-5, worst[1] / 1e-5, worst[2]))


@pytest.mark.parametrize("vps", [0, 2])
def test_update_dump_in_asynchronous_mode_is_consistent(vps):
    """Outside deterministic mode the record holds every executed update once (in a nondeterministic
    interleaving): the counts match mbir_stats and each voxel of iteration 1 appears exactly once;
    with voxel pairs no two consecutive records are both a pair's second update."""
    cfg = CONFIGS["cfg1"]
    case = make_case(cfg)
    g, _ = geoms(cfg)
    with M.Reconstructor(g, M.Prior(sigma=cfg.sigma, neighborhood=8),
                         M.Options(sv_side=cfg.sv_side, voxels_per_step=vps)) as r:
        r.set_sinogram(case.y, case.w)
        r.set_update_dump(10000)
        st = r.iterate(1)
        vox, t1, t2, dl, n = r.update_dump(10000)
        assert n == st["updates"] == cfg.n * cfg.n
        assert r.sizes()["voxels_per_step"] == (vps or 1)
        same = (vox & M.DUMP_SAME_STATE) != 0
        assert same.any() == (vps == 2) and not (same[1:] & same[:-1]).any()
        assert np.array_equal(np.sort(vox & (M.DUMP_SAME_STATE - 1)), np.arange(cfg.n * cfg.n))
        assert np.all(t2 > 0) and np.isfinite(t1).all() and np.isfinite(dl).all()
        st = r.iterate(1)
        n2 = r.update_dump(0)[4]
        assert n2 == st["updates"]
        r.set_update_dump(0)
        with pytest.raises(M.MbirError):
            r.update_dump(1)


@pytest.mark.parametrize("nz", [1, 3])
def test_device_rmse_hu_matches_oracle(nz):
    """mbir_rmse_hu (P:277 criterion, reading R12) against oracle.rmse_hu on the same float32
    images, host and device goldens, 1 HU = 2e-5 mm^-1 scale."""
    import torch
    cfg = WorkloadConfig("rm", 64, nz, 90, 96, 9, 26 if nz > 1 else 8, 0.002)
    g, _ = geoms(cfg)
    rng = np.random.default_rng(nz)
    x = rng.uniform(0, 0.04, (nz, 64, 64)).astype(np.float32)
    gold = (x + rng.normal(0, 3e-4, x.shape)).clip(0).astype(np.float32)
    with M.Reconstructor(g, M.Prior(neighborhood=cfg.nbhd), M.Options(sv_side=9)) as r:
        r.set_image(x)
        ref = O.rmse_hu(x, gold)
        assert r.rmse_hu(gold) == pytest.approx(ref, rel=1e-9)
        assert r.rmse_hu(torch.from_numpy(gold).cuda()) == pytest.approx(ref, rel=1e-9)
        assert r.rmse_hu(x + np.float32(2e-4)) == pytest.approx(10.0, rel=1e-4)
        assert r.rmse_hu(x) == 0.0


def _colour(sv, nsx):
    return (sv % nsx) % 2 + 2 * ((sv // nsx) % 2)


def test_scheduler_top_and_random_selection_and_colouring():
    """Alg3:17-23 / P:203-205 (reading R14): iteration 2 selects, in every slice, the ceil(25 %)
    SVs with the largest sum |delta| of their last visit (ties to the lower index), split into the
    four checkerboard colours in key order; iteration 3 selects a random ceil(25 %), the same SVs in
    every slice; no two SVs of one colour list touch (Fig. 3)."""
    cfg = WorkloadConfig("mini3d", 40, 4, 60, 64, 7, 26, 0.002)
    case = make_case(cfg)
    g, _ = geoms(cfg)
    with M.Reconstructor(g, M.Prior(sigma=cfg.sigma, neighborhood=26),
                         M.Options(sv_side=cfg.sv_side, zero_skip=0)) as r:
        r.set_sinogram(case.y, case.w)
        sz = r.sizes()
        nsv, nsx = sz["nsv"], sz["nsv_x"]
        nsel = int(np.ceil(0.25 * nsv))
        r.iterate(1)
        _, _, amount1 = r.schedule()
        # SVs whose every update clipped at 0 have amount 0: ties, broken by the lower index
        assert np.all(amount1 >= 0) and (amount1 == 0).any() and (amount1 > 0).sum() > nsel
        r.iterate(1)  # iteration 2: top 25 %
        tl, tc, _ = r.schedule()
        for z in range(cfg.nz):
            key = sorted(range(nsv), key=lambda s: (-float(amount1[z, s]), s))[:nsel]
            assert tc[z].sum() == nsel
            for c in range(4):
                got = list(tl[z, c, :tc[z, c]])
                assert got == [s for s in key if _colour(s, nsx) == c], (z, c)
        r.iterate(1)  # iteration 3: random 25 %
        tl, tc, _ = r.schedule()
        sel0 = None
        for z in range(cfg.nz):
            sel = []
            for c in range(4):
                lst = list(tl[z, c, :tc[z, c]])
                assert all(_colour(s, nsx) == c for s in lst)
                for a in lst:
                    for b in lst:
                        if a != b:
                            assert max(abs(a % nsx - b % nsx), abs(a // nsx - b // nsx)) >= 2
                sel += lst
            assert len(sel) == nsel and len(set(sel)) == nsel and all(0 <= s < nsv for s in sel)
            sel0 = sel0 or sorted(sel)
            assert sorted(sel) == sel0  # the same random subset in every slice (reading R14)
