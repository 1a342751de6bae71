"""ctypes binding of libmbir (include/mbir.h).  Argument marshalling only: every step of the
hot path runs in the library's sm_100a kernels.  There is no CPU fallback: importing the
functions fails loudly if libmbir.so has not been built (``__graft_entry__.build()``)."""
from __future__ import annotations

import ctypes as C
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libmbir.so")

MBIR_OK = 0
MBIR_EINVAL = -1
MBIR_ENOMEM = -2
MBIR_ECUDA = -3
MBIR_ESTATE = -4
MBIR_ENUMERIC = -5
MBIR_ENCCL = -6
MBIR_ENOTSUP = -7
MBIR_HOST = 0
MBIR_DEVICE = 1

# every symbol include/mbir.h declares (checked by tests/test_abi.py)
EXPORTS = (
    "mbir_default_options", "mbir_default_prior", "mbir_create", "mbir_set_sinogram",
    "mbir_set_image", "mbir_init_fbp", "mbir_reconstruct", "mbir_iterate", "mbir_get_image",
    "mbir_get_error_sinogram", "mbir_rmse_hu", "mbir_query_sizes", "mbir_get_sysmatrix",
    "mbir_get_sysmatrix_columns",
    "mbir_probe_update", "mbir_set_update_dump", "mbir_get_update_dump", "mbir_get_schedule",
    "mbir_link_slabs",
    "mbir_nccl_unique_id", "mbir_halo_plan", "mbir_destroy",
    "mbir_strerror", "mbir_last_error",
)


class mbir_geometry(C.Structure):
    _fields_ = [
        ("nx", C.c_int), ("ny", C.c_int),
        ("nz_local", C.c_int), ("z_offset", C.c_int), ("nz_total", C.c_int),
        ("dxy", C.c_double),
        ("nviews", C.c_int), ("nchannels", C.c_int),
        ("dchannel", C.c_double), ("center_offset", C.c_double),
        ("angles", C.POINTER(C.c_double)),
    ]


class mbir_prior(C.Structure):
    _fields_ = [("p", C.c_double), ("q", C.c_double), ("T", C.c_double), ("sigma", C.c_double),
                ("neighborhood", C.c_int), ("positivity", C.c_int)]


class mbir_options(C.Structure):
    _fields_ = [
        ("sv_side", C.c_int), ("sv_fraction", C.c_double), ("batch_svs", C.c_int),
        ("batch_threshold", C.c_int), ("zero_skip", C.c_int), ("quantize_A", C.c_int),
        ("seed", C.c_uint64), ("deterministic", C.c_int), ("cluster", C.c_int),
        ("zero_skip_period", C.c_int), ("voxels_per_step", C.c_int),
    ]


class mbir_dist(C.Structure):
    _fields_ = [("device", C.c_int), ("stream", C.c_void_p), ("rank", C.c_int),
                ("nranks", C.c_int), ("nccl_unique_id", C.c_void_p)]


class mbir_stats(C.Structure):
    _fields_ = [
        ("updates", C.c_int64), ("skipped", C.c_int64), ("sv_visits", C.c_int64),
        ("iterations", C.c_int64), ("equits", C.c_double), ("seconds", C.c_double),
        ("sum_abs_delta", C.c_double), ("launches", C.c_int64),
        ("kernel_seconds", C.c_double), ("kernel_launches", C.c_int64), ("sv_visits_empty", C.c_int64),
    ]

    def as_dict(self):
        return {k: getattr(self, k) for k, _ in self._fields_}


class mbir_sizes(C.Structure):
    _fields_ = [
        ("nsv_x", C.c_int), ("nsv_y", C.c_int), ("nsv", C.c_int), ("K", C.c_int),
        ("band_max", C.c_int), ("svb_rows", C.c_int), ("threads_per_cta", C.c_int), ("cluster", C.c_int), ("resident_ctas", C.c_int),
        ("smem_bytes", C.c_int), ("nnz", C.c_int64), ("a_bytes", C.c_int64),
        ("band_entries", C.c_int64), ("max_group", C.c_int), ("voxels_per_step", C.c_int),
    ]

    def as_dict(self):
        return {k: getattr(self, k) for k, _ in self._fields_}


_lib = None


def load(path: str = LIB_PATH):
    """Load libmbir.so (raises if it is missing -- no fallback).  MBIR_LIB may name another
    in-tree build of the same library (A/B kernel experiments)."""
    global _lib
    if _lib is not None:
        return _lib
    path = os.environ.get("MBIR_LIB", path)
    if not os.path.exists(path):
        raise ImportError(f"{path} not built: run `python -c 'import __graft_entry__ as g; g.build()'`")
    L = C.CDLL(path)
    H = C.c_void_p
    vp = C.c_void_p
    L.mbir_default_options.restype = None
    L.mbir_default_options.argtypes = [C.POINTER(mbir_options)]
    L.mbir_default_prior.restype = None
    L.mbir_default_prior.argtypes = [C.POINTER(mbir_prior)]
    L.mbir_create.restype = C.c_int
    L.mbir_create.argtypes = [C.POINTER(mbir_geometry), C.POINTER(mbir_prior),
                              C.POINTER(mbir_options), C.POINTER(mbir_dist), C.POINTER(H)]
    L.mbir_set_sinogram.restype = C.c_int
    L.mbir_set_sinogram.argtypes = [H, vp, vp, C.c_int]
    L.mbir_set_image.restype = C.c_int
    L.mbir_set_image.argtypes = [H, vp, C.c_int]
    L.mbir_init_fbp.restype = C.c_int
    L.mbir_init_fbp.argtypes = [H]
    L.mbir_reconstruct.restype = C.c_int
    L.mbir_reconstruct.argtypes = [H, C.c_double, C.POINTER(mbir_stats)]
    L.mbir_iterate.restype = C.c_int
    L.mbir_iterate.argtypes = [H, C.c_int, C.POINTER(mbir_stats)]
    L.mbir_get_image.restype = C.c_int
    L.mbir_get_image.argtypes = [H, vp, C.c_int]
    L.mbir_get_error_sinogram.restype = C.c_int
    L.mbir_get_error_sinogram.argtypes = [H, vp, C.c_int]
    L.mbir_rmse_hu.restype = C.c_int
    L.mbir_rmse_hu.argtypes = [H, vp, C.c_int, C.c_double, C.POINTER(C.c_double)]
    L.mbir_query_sizes.restype = C.c_int
    L.mbir_query_sizes.argtypes = [H, C.POINTER(mbir_sizes)]
    L.mbir_get_sysmatrix.restype = C.c_int
    L.mbir_get_sysmatrix.argtypes = [H, vp, vp, vp, vp, vp]
    L.mbir_get_sysmatrix_columns.restype = C.c_int
    L.mbir_get_sysmatrix_columns.argtypes = [H, vp, C.c_int, vp, vp, vp, vp, vp]
    L.mbir_probe_update.restype = C.c_int
    L.mbir_probe_update.argtypes = [H, vp, C.c_int, vp, vp, vp]
    L.mbir_link_slabs.restype = C.c_int
    L.mbir_link_slabs.argtypes = [C.POINTER(C.c_void_p), C.c_int]
    L.mbir_set_update_dump.restype = C.c_int
    L.mbir_set_update_dump.argtypes = [H, C.c_int64]
    L.mbir_get_update_dump.restype = C.c_int
    L.mbir_get_update_dump.argtypes = [H, C.c_int64, vp, vp, vp, vp, C.POINTER(C.c_int64)]
    L.mbir_get_schedule.restype = C.c_int
    L.mbir_get_schedule.argtypes = [H, vp, vp, vp]
    L.mbir_nccl_unique_id.restype = C.c_int
    L.mbir_nccl_unique_id.argtypes = [vp]
    L.mbir_halo_plan.restype = C.c_int
    L.mbir_halo_plan.argtypes = [C.c_int, C.c_int, C.c_int, C.c_int, C.c_int, vp]
    L.mbir_destroy.restype = None
    L.mbir_destroy.argtypes = [H]
    L.mbir_strerror.restype = C.c_char_p
    L.mbir_strerror.argtypes = [C.c_int]
    L.mbir_last_error.restype = C.c_char_p
    L.mbir_last_error.argtypes = [H]
    _lib = L
    return L


class MbirError(RuntimeError):
    def __init__(self, code: int, msg: str):
        super().__init__(f"{msg} (code {code})")
        self.code = code


def check(code: int, h=None, what: str = ""):
    if code != MBIR_OK:
        L = load()
        detail = L.mbir_last_error(h).decode() if h else ""
        raise MbirError(code, f"{what}: {L.mbir_strerror(code).decode()} {detail}".strip())
