"""ctypes wrapper around the sequential C oracle (oracle/oracle.c).

TEST INFRASTRUCTURE ONLY.  Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s
``cpu_baseline`` / ``--impl reference`` legs may import this module.  The product package
(``paper_conf_ppopp_sabnewkbrm17_b200``) never imports it; it shares no code with the CUDA path.

Every function mirrors one in ``oracle.h``; see that header for the PAPER.md citations
(Alg. 1 at P:99-113, P:115 randomised order / zero-skip, P:267-269 uint8 codec, Eq. 1 at P:351).
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB = os.path.join(_HERE, "liboracle.so")
MU_WATER = 0.02  # mm^-1, reading R12


def build(force: bool = False) -> str:
    src = os.path.join(_HERE, "oracle.c")
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(src):
        subprocess.check_call(["make", "-s", "-C", _HERE, "-B" if force else "liboracle.so"])
    return _LIB


class _Geom(C.Structure):
    _fields_ = [
        ("nx", C.c_int), ("ny", C.c_int), ("nz", C.c_int),
        ("dxy", C.c_double),
        ("nviews", C.c_int), ("nchannels", C.c_int),
        ("dchannel", C.c_double), ("center_offset", C.c_double),
        ("angles", C.POINTER(C.c_double)),
    ]


class _Prior(C.Structure):
    _fields_ = [
        ("p", C.c_double), ("q", C.c_double), ("T", C.c_double), ("sigma", C.c_double),
        ("nbhd", C.c_int), ("positivity", C.c_int),
    ]


class _Stats(C.Structure):
    _fields_ = [("updates", C.c_int64), ("skipped", C.c_int64), ("sum_abs_delta", C.c_double)]


_lib = None


def lib():
    global _lib
    if _lib is None:
        build()
        L = C.CDLL(_LIB)
        dp, ip, lp = C.POINTER(C.c_double), C.POINTER(C.c_int32), C.POINTER(C.c_int64)
        u8p = C.POINTER(C.c_uint8)
        G, P = C.POINTER(_Geom), C.POINTER(_Prior)
        L.orc_strip_pixel_area.restype = C.c_double
        L.orc_strip_pixel_area.argtypes = [C.c_double] * 7
        L.orc_view_angle.restype = C.c_double
        L.orc_view_angle.argtypes = [G, C.c_int]
        L.orc_sysmatrix_column.restype = C.c_int
        L.orc_sysmatrix_column.argtypes = [G, C.c_int, C.c_int, C.c_int, ip, ip, dp]
        L.orc_sysmatrix_build.restype = C.c_int
        L.orc_sysmatrix_build.argtypes = [G, C.c_int, ip, ip, dp]
        L.orc_quantize_column.restype = C.c_double
        L.orc_quantize_column.argtypes = [dp, ip, C.c_int, C.c_int, u8p]
        L.orc_rho.restype = C.c_double
        L.orc_rho.argtypes = [C.c_double, P]
        L.orc_phi.restype = C.c_double
        L.orc_phi.argtypes = [C.c_double, P]
        L.orc_nbr_weight.restype = C.c_double
        L.orc_nbr_weight.argtypes = [C.c_int, C.c_int, C.c_int, C.c_int]
        L.orc_voxel_update.restype = None
        L.orc_voxel_update.argtypes = [G, P, C.c_int, ip, ip, dp, dp, dp, dp, C.c_int64,
                                       C.c_int, dp, dp, dp]
        L.orc_icd_run.restype = C.c_int64
        L.orc_icd_run.argtypes = [G, P, C.c_int, ip, ip, dp, dp, dp, dp, C.c_int, C.c_int,
                                  C.c_uint64, C.c_int, C.c_int, lp, C.c_int64, dp, C.c_int64,
                                  C.POINTER(_Stats)]
        L.orc_icd_run_zpar.restype = C.c_int
        L.orc_icd_run_zpar.argtypes = [G, P, C.c_int, ip, ip, dp, dp, dp, dp, C.c_int, C.c_int,
                                       C.c_uint64, C.c_int, C.c_int, C.c_int, C.POINTER(_Stats)]
        L.orc_error_sinogram.restype = None
        L.orc_error_sinogram.argtypes = [G, C.c_int, ip, ip, dp, dp, dp, dp]
        L.orc_cost.restype = C.c_double
        L.orc_cost.argtypes = [G, P, C.c_int, ip, ip, dp, dp, dp, dp]
        L.orc_rmse_hu.restype = C.c_double
        L.orc_rmse_hu.argtypes = [dp, dp, C.c_int64, C.c_double]
        _lib = L
    return _lib


def _p(a, t):
    return a.ctypes.data_as(C.POINTER(t))


@dataclass
class Geometry:
    nx: int
    ny: int
    nz: int
    dxy: float
    nviews: int
    nchannels: int
    dchannel: float
    center_offset: float = 0.0
    angles: np.ndarray | None = None

    def c(self):
        g = _Geom(self.nx, self.ny, self.nz, self.dxy, self.nviews, self.nchannels,
                  self.dchannel, self.center_offset, None)
        if self.angles is not None:
            self._ang = np.ascontiguousarray(self.angles, dtype=np.float64)
            g.angles = _p(self._ang, C.c_double)
        return g


@dataclass
class Prior:
    p: float = 1.2
    q: float = 2.0
    T: float = 1.0
    sigma: float = 0.01
    nbhd: int = 8
    positivity: int = 1

    def c(self):
        return _Prior(self.p, self.q, self.T, self.sigma, self.nbhd, self.positivity)


@dataclass
class SysMatrix:
    """Oracle's own sparse A: first/count [nx*ny, V], vals [nx*ny, V, K] (double)."""
    first: np.ndarray
    count: np.ndarray
    vals: np.ndarray
    K: int
    maxcount: int


def strip_pixel_area(cx, cy, d, c, s, tlo, thi):
    return lib().orc_strip_pixel_area(cx, cy, d, c, s, tlo, thi)


def view_angle(g: Geometry, k: int) -> float:
    gc = g.c()
    return lib().orc_view_angle(C.byref(gc), k)


def sysmatrix_column(g: Geometry, ix: int, iy: int, K: int = 4):
    V = g.nviews
    first = np.zeros(V, np.int32)
    count = np.zeros(V, np.int32)
    vals = np.zeros((V, K), np.float64)
    gc = g.c()
    m = lib().orc_sysmatrix_column(C.byref(gc), ix, iy, K, _p(first, C.c_int32),
                                   _p(count, C.c_int32), _p(vals, C.c_double))
    return first, count, vals, m


def sysmatrix(g: Geometry, K: int = 4) -> SysMatrix:
    n = g.nx * g.ny
    first = np.zeros((n, g.nviews), np.int32)
    count = np.zeros((n, g.nviews), np.int32)
    vals = np.zeros((n, g.nviews, K), np.float64)
    gc = g.c()
    m = lib().orc_sysmatrix_build(C.byref(gc), K, _p(first, C.c_int32), _p(count, C.c_int32),
                                  _p(vals, C.c_double))
    if m > K:
        raise ValueError(f"geometry needs K >= {m}")
    return SysMatrix(first, count, vals, K, m)


def quantize_column(vals: np.ndarray, count: np.ndarray):
    """Returns (codes uint8 [V,K], amax)."""
    vals = np.ascontiguousarray(vals, np.float64)
    count = np.ascontiguousarray(count, np.int32)
    V, K = vals.shape
    codes = np.zeros((V, K), np.uint8)
    amax = lib().orc_quantize_column(_p(vals, C.c_double), _p(count, C.c_int32), V, K,
                                     _p(codes, C.c_uint8))
    return codes, amax


def quantize(A: SysMatrix):
    """Per-voxel uint8 codes and amax for the whole A; also the dequantised A (double)."""
    n, V, K = A.vals.shape
    codes = np.zeros((n, V, K), np.uint8)
    amax = np.zeros(n, np.float64)
    for j in range(n):
        codes[j], amax[j] = quantize_column(A.vals[j], A.count[j])
    deq = codes.astype(np.float64) * (amax / 255.0)[:, None, None]
    return codes, amax, SysMatrix(A.first, A.count, deq, K, A.maxcount)


def rho(delta: float, pr: Prior) -> float:
    pc = pr.c()
    return lib().orc_rho(delta, C.byref(pc))


def phi(delta: float, pr: Prior) -> float:
    pc = pr.c()
    return lib().orc_phi(delta, C.byref(pc))


def nbr_weight(dx, dy, dz, nbhd):
    return lib().orc_nbr_weight(dx, dy, dz, nbhd)


def error_sinogram(g: Geometry, A: SysMatrix, y: np.ndarray, x: np.ndarray) -> np.ndarray:
    y = np.ascontiguousarray(y, np.float64)
    x = np.ascontiguousarray(x, np.float64)
    e = np.empty_like(y)
    gc = g.c()
    lib().orc_error_sinogram(C.byref(gc), A.K, _p(A.first, C.c_int32), _p(A.count, C.c_int32),
                             _p(A.vals, C.c_double), _p(y, C.c_double), _p(x, C.c_double),
                             _p(e, C.c_double))
    return e


def voxel_update(g: Geometry, pr: Prior, A: SysMatrix, w, x, e, j: int, apply: bool = False):
    """Alg. 1 on voxel j (flat index).  x, e are modified in place iff apply."""
    assert x.dtype == np.float64 and x.flags.c_contiguous
    assert e.dtype == np.float64 and e.flags.c_contiguous
    w = np.ascontiguousarray(w, np.float64)
    plane = g.nx * g.ny
    jj = j % plane
    t1, t2, dl = C.c_double(), C.c_double(), C.c_double()
    gc, pc = g.c(), pr.c()
    first = np.ascontiguousarray(A.first[jj])
    count = np.ascontiguousarray(A.count[jj])
    vals = np.ascontiguousarray(A.vals[jj])
    lib().orc_voxel_update(C.byref(gc), C.byref(pc), A.K, _p(first, C.c_int32),
                           _p(count, C.c_int32), _p(vals, C.c_double), _p(w, C.c_double),
                           _p(x, C.c_double), _p(e, C.c_double), j, int(apply),
                           C.byref(t1), C.byref(t2), C.byref(dl))
    return t1.value, t2.value, dl.value


def icd_run(g: Geometry, pr: Prior, A: SysMatrix, w, x, e, n_equits: int, *, first_sweep=1,
            seed=3000, zero_skip=True, zero_skip_period=0, order=None, dump=0):
    """Sequential ICD.  x, e (float64, contiguous) updated in place.
    zero_skip_period > 0: sweeps numbered by a multiple of it run without zero-skipping
    (reading R9).  Returns (stats dict, dump array [n,4] of (j, theta1, theta2, delta))."""
    assert x.dtype == np.float64 and x.flags.c_contiguous
    assert e.dtype == np.float64 and e.flags.c_contiguous
    w = np.ascontiguousarray(w, np.float64)
    st = _Stats()
    gc, pc = g.c(), pr.c()
    order_arr = None
    if order is not None:
        order_arr = np.ascontiguousarray(order, np.int64)
    dbuf = np.zeros((max(dump, 1), 4), np.float64)
    n = lib().orc_icd_run(C.byref(gc), C.byref(pc), A.K, _p(A.first, C.c_int32),
                          _p(A.count, C.c_int32), _p(A.vals, C.c_double), _p(w, C.c_double),
                          _p(x, C.c_double), _p(e, C.c_double), n_equits, first_sweep,
                          C.c_uint64(seed), int(zero_skip), int(zero_skip_period),
                          _p(order_arr, C.c_int64) if order_arr is not None else None,
                          len(order_arr) if order_arr is not None else 0,
                          _p(dbuf, C.c_double) if dump else None, dump, C.byref(st))
    if n < 0:
        raise MemoryError("oracle icd_run")
    return ({"updates": st.updates, "skipped": st.skipped, "sum_abs_delta": st.sum_abs_delta},
            dbuf[:n] if dump else None)


def icd_run_zpar(g: Geometry, pr: Prior, A: SysMatrix, w, x, e, n_equits: int, *, first_sweep=1,
                 seed=3000, zero_skip=False, zero_skip_period=0, threads=None):
    """Sequential ICD with the slices of one z-parity on several host threads (an exact
    serialisation, see oracle.h orc_icd_run_zpar).  x, e updated in place.  Returns stats."""
    assert x.dtype == np.float64 and x.flags.c_contiguous
    assert e.dtype == np.float64 and e.flags.c_contiguous
    w = np.ascontiguousarray(w, np.float64)
    st = _Stats()
    gc, pc = g.c(), pr.c()
    nt = threads or (os.cpu_count() or 1)
    r = lib().orc_icd_run_zpar(C.byref(gc), C.byref(pc), A.K, _p(A.first, C.c_int32),
                               _p(A.count, C.c_int32), _p(A.vals, C.c_double), _p(w, C.c_double),
                               _p(x, C.c_double), _p(e, C.c_double), n_equits, first_sweep,
                               C.c_uint64(seed), int(zero_skip), int(zero_skip_period), nt,
                               C.byref(st))
    if r < 0:
        raise MemoryError("oracle icd_run_zpar")
    return {"updates": st.updates, "skipped": st.skipped, "sum_abs_delta": st.sum_abs_delta,
            "threads": nt}


def cost(g: Geometry, pr: Prior, A: SysMatrix, y, w, x) -> float:
    y = np.ascontiguousarray(y, np.float64)
    w = np.ascontiguousarray(w, np.float64)
    x = np.ascontiguousarray(x, np.float64)
    gc, pc = g.c(), pr.c()
    return lib().orc_cost(C.byref(gc), C.byref(pc), A.K, _p(A.first, C.c_int32),
                          _p(A.count, C.c_int32), _p(A.vals, C.c_double), _p(y, C.c_double),
                          _p(w, C.c_double), _p(x, C.c_double))


def rmse_hu(a, b, mu_water: float = MU_WATER) -> float:
    a = np.ascontiguousarray(a, np.float64).ravel()
    b = np.ascontiguousarray(b, np.float64).ravel()
    return lib().orc_rmse_hu(_p(a, C.c_double), _p(b, C.c_double), a.size, mu_water)


def fbp(g: Geometry, y, positivity: bool = True) -> np.ndarray:
    """Filtered back-projection of y [nz][V][M] (the optional initial image of mbir_init_fbp;
    not part of the paper's method, reading R23), in float64, written from the textbook
    definition (Kak & Slaney, ch. 3, eqs. 61-63): q_k = dc * (h * p_k) with the band-limited ramp
    h(0) = 1/(4 dc^2), h(n dc) = -1/(pi^2 n^2 dc^2) for odd n, 0 for even n != 0 (full linear
    convolution, np.convolve); f(x, y) = (pi / V) sum_k q_k(x cos th_k + y sin th_k), linear
    interpolation between channel centres t0 + (m + 1/2) dc, zero outside the detector.
    Returns [nz][ny][nx], clipped at 0 when positivity."""
    y = np.asarray(y, np.float64)
    V, M = g.nviews, g.nchannels
    dc = g.dchannel
    n = np.arange(-(M - 1), M)
    h = np.zeros(n.size)
    h[n == 0] = 1.0 / (4 * dc * dc)
    odd = n % 2 != 0
    h[odd] = -1.0 / (np.pi ** 2 * n[odd].astype(np.float64) ** 2 * dc * dc)
    th = np.asarray(g.angles, np.float64) if g.angles is not None else np.arange(V) * np.pi / V
    t0 = -0.5 * M * dc + g.center_offset * dc
    xc = (np.arange(g.nx) - 0.5 * (g.nx - 1)) * g.dxy
    yc = (np.arange(g.ny) - 0.5 * (g.ny - 1)) * g.dxy
    X, Y = np.meshgrid(xc, yc)  # [iy][ix]
    out = np.zeros((y.shape[0], g.ny, g.nx))
    for z in range(y.shape[0]):
        for k in range(V):
            q = dc * np.convolve(y[z, k], h)[M - 1: 2 * M - 1]
            u = (X * np.cos(th[k]) + Y * np.sin(th[k]) - t0) / dc - 0.5
            m = np.floor(u).astype(np.int64)
            f = u - m
            qa = np.where((m >= 0) & (m < M), q[np.clip(m, 0, M - 1)], 0.0)
            qb = np.where((m + 1 >= 0) & (m + 1 < M), q[np.clip(m + 1, 0, M - 1)], 0.0)
            out[z] += qa + f * (qb - qa)
    out *= np.pi / V
    return np.maximum(out, 0.0) if positivity else out
