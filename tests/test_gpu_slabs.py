"""The z-slab partition of the multi-GPU path verified on one
GPU: 2 and 4 handles own consecutive slabs of one volume and exchange halo slices after every
z-parity half exactly as mbir_halo_plan schedules it -- by device-to-device copies (test hook
mbir_link_slabs) instead of NCCL.  Same-parity slices share no data and the phases run z-parity
major, so in deterministic mode the slab run must equal the single-handle run BIT FOR BIT,
including zero-skipping across slab boundaries and the 26-neighbourhood prior at them."""
import threading

import numpy as np
import pytest

import paper_conf_ppopp_sabnewkbrm17_b200 as M
from synth import WorkloadConfig, make_case

pytestmark = pytest.mark.gpu


def _single(cfg, case, opts, iters, x0):
    g = M.Geometry(cfg.n, cfg.n, cfg.nz, cfg.dxy, cfg.nviews, cfg.nchannels, cfg.dchannel)
    with M.Reconstructor(g, M.Prior(sigma=cfg.sigma, neighborhood=26), opts) as r:
        r.set_sinogram(case.y, case.w)
        r.set_image(x0)
        sts = [r.iterate(1) for _ in range(iters)]
        return r.image(), r.error_sinogram(), sum(s["updates"] for s in sts)


def _slabs(cfg, case, opts, iters, x0, nsl):
    per = cfg.nz // nsl
    rs = []
    for i in range(nsl):
        g = M.Geometry(cfg.n, cfg.n, per, cfg.dxy, cfg.nviews, cfg.nchannels, cfg.dchannel,
                       z_offset=i * per, nz_total=cfg.nz)
        rs.append(M.Reconstructor(g, M.Prior(sigma=cfg.sigma, neighborhood=26), opts, rank=i, nranks=nsl))
    M.mbir_link_slabs([r.h for r in rs])
    out, err = [None] * nsl, []

    def drive(i):
        try:
            r = rs[i]
            sl = slice(i * per, (i + 1) * per)
            r.set_sinogram(np.ascontiguousarray(case.y[sl]), np.ascontiguousarray(case.w[sl]))
            r.set_image(np.ascontiguousarray(x0[sl]))  # collective: the halo exchange
            upd = sum(r.iterate(1)["updates"] for _ in range(iters))  # collective per half
            out[i] = (r.image(), r.error_sinogram(), upd)
        except Exception as e:  # pragma: no cover - surfaced below
            err.append(e)

    th = [threading.Thread(target=drive, args=(i,)) for i in range(nsl)]
    for t in th:
        t.start()
    for t in th:
        t.join(timeout=600)
    for r in rs:
        r.close()
    assert not err, err
    return (np.concatenate([o[0] for o in out]), np.concatenate([o[1] for o in out]), sum(o[2] for o in out))


@pytest.mark.parametrize("nsl", [2, 4])
@pytest.mark.parametrize("zero_skip", [0, 1])
def test_linked_slabs_equal_single_handle_bitwise(nsl, zero_skip):
    cfg = WorkloadConfig("slab3d", 40, 8, 60, 64, 7, 26, 0.002, phantom="baggage")
    case = make_case(cfg, 101)
    # from x0 = 0 (e = y exactly: a warm start's forward projection accumulates with atomics, whose
    # order is not reproducible bit for bit); baggage scenes leave exact zeros in the air, so
    # iterations >= 2 zero-skip across the slab boundaries
    x0 = np.zeros((cfg.nz, cfg.n, cfg.n), np.float32)
    opts = M.Options(sv_side=cfg.sv_side, deterministic=1, zero_skip=zero_skip)
    xs, es, us = _single(cfg, case, opts, 4, x0)
    xl, el, ul = _slabs(cfg, case, opts, 4, x0, nsl)
    assert us == ul
    np.testing.assert_array_equal(xl, xs)
    np.testing.assert_array_equal(el, es)
    assert xs.max() > 0 and (xs == 0).mean() > 0.2


def test_link_slabs_argument_checks():
    cfg = WorkloadConfig("slab3d", 40, 8, 60, 64, 7, 26, 0.002)
    mk = lambda i, z0: M.Reconstructor(M.Geometry(cfg.n, cfg.n, 4, cfg.dxy, cfg.nviews, cfg.nchannels,
                                                  cfg.dchannel, z_offset=z0, nz_total=8),
                                       M.Prior(neighborhood=26), M.Options(sv_side=7), rank=i, nranks=2)
    a, b = mk(0, 0), mk(1, 4)
    with pytest.raises(M.MbirError):
        M.mbir_link_slabs([b.h, a.h])  # wrong rank order
    with pytest.raises(M.MbirError) as ei:
        a.set_image(None)  # collective before linking: no NCCL, no link
    assert ei.value.code == -4
    M.mbir_link_slabs([a.h, b.h])
    with pytest.raises(M.MbirError):
        M.mbir_link_slabs([a.h, b.h])  # already linked
    a.close()
    b.close()
