"""ctypes wrapper around the PSV-ICD CPU comparison build (psvicd.c; Alg. 2, P:131-143;
SURVEY 8(f) NEXT-4).

A baseline, not the product and not the oracle: bench.py's `psv_icd` leg and
tests/test_psvicd.py use it.  It takes the system matrix as (first, count, vals) arrays, which
its callers take from ``oracle.sysmatrix`` (test infrastructure), dequantised to the codes the GPU
path runs with.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB = os.path.join(_HERE, "libpsvicd.so")


class _Geom(C.Structure):
    _fields_ = [("nx", C.c_int), ("ny", C.c_int), ("nz", C.c_int), ("nviews", C.c_int), ("nchannels", C.c_int)]


class _Prior(C.Structure):
    _fields_ = [("p", C.c_double), ("q", C.c_double), ("T", C.c_double), ("sigma", C.c_double),
                ("nbhd", C.c_int), ("positivity", C.c_int)]


class _Stats(C.Structure):
    _fields_ = [("updates", C.c_int64), ("skipped", C.c_int64), ("sum_abs_delta", C.c_double),
                ("seconds", C.c_double), ("iterations", C.c_int)]


_lib = None


def build(force: bool = False) -> str:
    src = os.path.join(_HERE, "psvicd.c")
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(src):
        subprocess.check_call(["make", "-s", "-C", _HERE, "-B" if force else "libpsvicd.so"])
    return _LIB


def lib():
    global _lib
    if _lib is None:
        build()
        L = C.CDLL(_LIB)
        ip, dp, fp = C.POINTER(C.c_int32), C.POINTER(C.c_double), C.POINTER(C.c_float)
        L.psv_create.restype = C.c_int
        L.psv_create.argtypes = [C.POINTER(_Geom), C.POINTER(_Prior), C.c_int, ip, ip, dp, C.c_int,
                                 C.POINTER(C.c_void_p)]
        L.psv_iterate.restype = C.c_int
        L.psv_iterate.argtypes = [C.c_void_p, fp, fp, fp, C.c_int, C.c_double, C.c_uint64, C.c_int, C.c_int,
                                  C.c_int, C.c_int, C.POINTER(_Stats)]
        L.psv_destroy.restype = None
        L.psv_destroy.argtypes = [C.c_void_p]
        _lib = L
    return _lib


def _p(a, t):
    return a.ctypes.data_as(C.POINTER(t))


class PSVICD:
    """PSV-ICD over one volume.  x [nz][ny][nx] and e [nz][V][M] are float32 arrays owned by the
    caller and updated in place by iterate()."""

    def __init__(self, nx, ny, nz, nviews, nchannels, A, *, sigma, p=1.2, q=2.0, T=1.0, nbhd=8,
                 positivity=1, sv_side=13):
        self._h = None
        self._g = _Geom(nx, ny, nz, nviews, nchannels)
        self._pr = _Prior(p, q, T, sigma, nbhd, positivity)
        self.shape = (nz, ny, nx)
        first = np.ascontiguousarray(A.first, np.int32)
        count = np.ascontiguousarray(A.count, np.int32)
        vals = np.ascontiguousarray(A.vals, np.float64)
        h = C.c_void_p()
        rc = lib().psv_create(C.byref(self._g), C.byref(self._pr), int(A.K), _p(first, C.c_int32),
                              _p(count, C.c_int32), _p(vals, C.c_double), int(sv_side), C.byref(h))
        if rc != 0:
            raise ValueError(f"psv_create failed ({rc})")
        self._h = h

    def iterate(self, w, x, e, n_iters=1, *, frac=0.2, seed=11, zero_skip=True, zero_skip_period=4,
                threads=None, raster=False):
        """Alg. 2 iterations (frac = the share of SVs after iteration 1; the paper's 20 %)."""
        for a in (w, x, e):
            assert a.dtype == np.float32 and a.flags.c_contiguous
        st = _Stats()
        nt = threads or (os.cpu_count() or 1)
        rc = lib().psv_iterate(self._h, _p(w, C.c_float), _p(x, C.c_float), _p(e, C.c_float), int(n_iters),
                               float(frac), C.c_uint64(seed), int(zero_skip), int(zero_skip_period), int(nt),
                               int(raster), C.byref(st))
        if rc != 0:
            raise RuntimeError(f"psv_iterate failed ({rc})")
        return {"updates": st.updates, "skipped": st.skipped, "sum_abs_delta": st.sum_abs_delta,
                "seconds": st.seconds, "iterations": st.iterations, "threads": nt}

    def close(self):
        if self._h:
            lib().psv_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass
