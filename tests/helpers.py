"""Test-side helpers shared by the GPU parity tests (no method arithmetic of the CUDA path)."""
import numpy as np

import oracle as O
import paper_conf_ppopp_sabnewkbrm17_b200 as M


def geoms(cfg, nz=None):
    nz = cfg.nz if nz is None else nz
    g = M.Geometry(cfg.n, cfg.n, nz, cfg.dxy, cfg.nviews, cfg.nchannels, cfg.dchannel)
    og = O.Geometry(cfg.n, cfg.n, nz, cfg.dxy, cfg.nviews, cfg.nchannels, cfg.dchannel)
    return g, og


def deterministic_order(n, nz, side, nbhd):
    """Global voxel order of the library's deterministic debug mode (include/mbir.h
    mbir_options.deterministic): z-parity half (3-D prior only), colour, SV rank within the
    colour (index order), slice, raster within the SV -- written from the documented contract,
    not from the CUDA code."""
    nsx = (n + side - 1) // side
    parities = [0, 1] if (nbhd == 26 and nz > 1) else [None]
    order = []
    for zp in parities:
        for colour in range(4):
            svs = [sv for sv in range(nsx * nsx) if ((sv % nsx) & 1) + 2 * ((sv // nsx) & 1) == colour]
            for sv in svs:
                bx, by = sv % nsx, sv // nsx
                for z in range(nz):
                    if zp is not None and z % 2 != zp:
                        continue
                    for ly in range(side):
                        for lx in range(side):
                            ix, iy = bx * side + lx, by * side + ly
                            if ix < n and iy < n:
                                order.append((z * n + iy) * n + ix)
    return np.array(order, np.int64)
