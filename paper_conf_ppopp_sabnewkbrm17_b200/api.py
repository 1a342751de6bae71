"""Thin Python binding of the libmbir C-ABI (include/mbir.h), same names as the C calls.

Buffers may be numpy arrays (host), torch CPU tensors (host) or torch CUDA tensors (device);
each must be float32, C-contiguous and of the documented shape.  PyTorch is only the
allocator / stream / process-group provider; all computation happens in libmbir's kernels.
"""
from __future__ import annotations

import ctypes as C
from dataclasses import dataclass

import numpy as np

from . import _lib as L

__all__ = [
    "Geometry", "Prior", "Options", "mbir_create", "mbir_set_sinogram", "mbir_set_image",
    "mbir_reconstruct", "mbir_iterate", "mbir_get_image", "mbir_get_error_sinogram",
    "mbir_rmse_hu", "mbir_query_sizes", "mbir_get_sysmatrix", "mbir_get_sysmatrix_columns",
    "mbir_probe_update", "mbir_set_update_dump", "mbir_get_update_dump", "mbir_get_schedule",
    "mbir_link_slabs", "mbir_nccl_unique_id", "mbir_destroy", "Reconstructor",
]


@dataclass
class Geometry:
    """mbir_geometry (readings R4-R5)."""
    nx: int
    ny: int
    nz_local: int
    dxy: float
    nviews: int
    nchannels: int
    dchannel: float
    center_offset: float = 0.0
    z_offset: int = 0
    nz_total: int = 0
    angles: np.ndarray | None = None

    def c(self) -> L.mbir_geometry:
        g = L.mbir_geometry(self.nx, self.ny, self.nz_local, self.z_offset,
                            self.nz_total or self.nz_local, self.dxy, self.nviews, self.nchannels,
                            self.dchannel, self.center_offset, None)
        if self.angles is not None:
            self._ang = np.ascontiguousarray(self.angles, np.float64)
            g.angles = self._ang.ctypes.data_as(C.POINTER(C.c_double))
        return g


@dataclass
class Prior:
    """mbir_prior: q-GGMRF (reading R1)."""
    p: float = 1.2
    q: float = 2.0
    T: float = 1.0
    sigma: float = 0.005
    neighborhood: int = 26
    positivity: int = 1

    def c(self) -> L.mbir_prior:
        return L.mbir_prior(self.p, self.q, self.T, self.sigma, self.neighborhood, self.positivity)


@dataclass
class Options:
    """mbir_options (Alg. 3, Table 1)."""
    sv_side: int = 9
    sv_fraction: float = 0.25
    batch_svs: int = 0
    batch_threshold: int = -1
    zero_skip: int = 1
    quantize_A: int = 1
    seed: int = 3000
    deterministic: int = 0
    cluster: int = 0  # update-kernel CTAs per SV task: 0 (auto) = 1, or 2 (a cluster splits the views)
    zero_skip_period: int = 4  # every n-th iteration without zero-skip (reading R9); 0 = never
    voxels_per_step: int = 0  # voxels of an SV per kernel step: 0 auto (= 1), 1, or 2 (voxel pairs)

    def c(self) -> L.mbir_options:
        return L.mbir_options(self.sv_side, self.sv_fraction, self.batch_svs,
                              self.batch_threshold, self.zero_skip, self.quantize_A, self.seed,
                              self.deterministic, self.cluster, self.zero_skip_period,
                              self.voxels_per_step)


def _buf(a, n: int | None = None, dtype=np.float32, writable=False):
    """(pointer, where) for a numpy array or torch tensor."""
    if hasattr(a, "data_ptr"):  # torch tensor
        import torch
        want = {np.float32: torch.float32, np.int32: torch.int32, np.uint8: torch.uint8,
                np.int64: torch.int64}[dtype]
        if a.dtype != want or not a.is_contiguous():
            raise ValueError(f"tensor must be contiguous {want}")
        if n is not None and a.numel() != n:
            raise ValueError(f"tensor has {a.numel()} elements, expected {n}")
        return C.c_void_p(a.data_ptr()), (L.MBIR_DEVICE if a.is_cuda else L.MBIR_HOST)
    if not isinstance(a, np.ndarray) or a.dtype != dtype or not a.flags.c_contiguous:
        raise ValueError(f"array must be a C-contiguous {np.dtype(dtype).name} ndarray")
    if writable and not a.flags.writeable:
        raise ValueError("array must be writable")
    if n is not None and a.size != n:
        raise ValueError(f"array has {a.size} elements, expected {n}")
    return C.c_void_p(a.ctypes.data), L.MBIR_HOST


def mbir_nccl_unique_id() -> bytes:
    buf = (C.c_char * 128)()
    L.check(L.load().mbir_nccl_unique_id(buf), None, "mbir_nccl_unique_id")
    return bytes(buf)


def _torch_current_stream(device: int):
    """torch's current CUDA stream on `device` (as a cudaStream_t), if torch is already in use
    with CUDA: the library then orders its work after the torch kernels that produced its device
    inputs (mbir.h: device buffers must be ready on the handle's stream).  None otherwise (the
    library creates its own stream)."""
    import sys
    torch = sys.modules.get("torch")
    if torch is None or not torch.cuda.is_available():
        return None
    return torch.cuda.current_stream(device).cuda_stream or None


def mbir_create(g: Geometry, p: Prior | None = None, o: Options | None = None, *, device: int = 0,
                stream: int | None = None, rank: int = 0, nranks: int = 1,
                nccl_id: bytes | None = None):
    lib = L.load()
    if stream is None:
        stream = _torch_current_stream(device)
    gc = g.c()
    pc = (p or Prior()).c()
    oc = (o or Options()).c()
    idbuf = C.create_string_buffer(nccl_id, 128) if nccl_id is not None else None
    dc = L.mbir_dist(device, C.c_void_p(stream) if stream else None, rank, nranks,
                     C.cast(idbuf, C.c_void_p) if idbuf is not None else None)
    h = C.c_void_p()
    code = lib.mbir_create(C.byref(gc), C.byref(pc), C.byref(oc), C.byref(dc), C.byref(h))
    L.check(code, None, "mbir_create")
    return h


def _n_sino(g: Geometry):
    return g.nz_local * g.nviews * g.nchannels


def _n_img(g: Geometry):
    return g.nz_local * g.ny * g.nx


def mbir_set_sinogram(h, g: Geometry, y, w):
    py, wy = _buf(y, _n_sino(g))
    pw, ww = _buf(w, _n_sino(g))
    if wy != ww:
        raise ValueError("y and w must both be host or both be device buffers")
    L.check(L.load().mbir_set_sinogram(h, py, pw, wy), h, "mbir_set_sinogram")


def mbir_set_image(h, g: Geometry, x0=None):
    if x0 is None:
        L.check(L.load().mbir_set_image(h, None, L.MBIR_HOST), h, "mbir_set_image")
        return
    px, where = _buf(x0, _n_img(g))
    L.check(L.load().mbir_set_image(h, px, where), h, "mbir_set_image")


def mbir_init_fbp(h):
    L.check(L.load().mbir_init_fbp(h), h, "mbir_init_fbp")


def mbir_reconstruct(h, equits: float) -> dict:
    st = L.mbir_stats()
    L.check(L.load().mbir_reconstruct(h, float(equits), C.byref(st)), h, "mbir_reconstruct")
    return st.as_dict()


def mbir_iterate(h, n_iterations: int) -> dict:
    st = L.mbir_stats()
    L.check(L.load().mbir_iterate(h, int(n_iterations), C.byref(st)), h, "mbir_iterate")
    return st.as_dict()


def mbir_get_image(h, g: Geometry, out=None):
    if out is None:
        out = np.empty((g.nz_local, g.ny, g.nx), np.float32)
    p, where = _buf(out, _n_img(g), writable=True)
    L.check(L.load().mbir_get_image(h, p, where), h, "mbir_get_image")
    return out


def mbir_get_error_sinogram(h, g: Geometry, out=None):
    if out is None:
        out = np.empty((g.nz_local, g.nviews, g.nchannels), np.float32)
    p, where = _buf(out, _n_sino(g), writable=True)
    L.check(L.load().mbir_get_error_sinogram(h, p, where), h, "mbir_get_error_sinogram")
    return out


def mbir_rmse_hu(h, g: Geometry, golden, mu_water: float = 0.02) -> float:
    p, where = _buf(golden, _n_img(g))
    out = C.c_double()
    L.check(L.load().mbir_rmse_hu(h, p, where, mu_water, C.byref(out)), h, "mbir_rmse_hu")
    return out.value


def mbir_query_sizes(h) -> dict:
    s = L.mbir_sizes()
    L.check(L.load().mbir_query_sizes(h, C.byref(s)), h, "mbir_query_sizes")
    return s.as_dict()


def mbir_get_sysmatrix(h, g: Geometry):
    """Plain-layout export: first, count [ny*nx, V] int32; values [ny*nx, V, 4] float32;
    codes [ny*nx, V, 4] uint8; scales [ny*nx] float32."""
    n, V = g.nx * g.ny, g.nviews
    first = np.empty((n, V), np.int32)
    count = np.empty((n, V), np.int32)
    vals = np.empty((n, V, 4), np.float32)
    codes = np.empty((n, V, 4), np.uint8)
    scales = np.empty(n, np.float32)
    L.check(L.load().mbir_get_sysmatrix(h, first.ctypes.data, count.ctypes.data, vals.ctypes.data,
                                        codes.ctypes.data, scales.ctypes.data), h,
            "mbir_get_sysmatrix")
    return first, count, vals, codes, scales


def mbir_get_sysmatrix_columns(h, g: Geometry, voxels):
    """Like mbir_get_sysmatrix for the listed in-slice voxels only (rows in list order)."""
    vox = np.ascontiguousarray(voxels, np.int64)
    n, V = vox.size, g.nviews
    first = np.empty((n, V), np.int32)
    count = np.empty((n, V), np.int32)
    vals = np.empty((n, V, 4), np.float32)
    codes = np.empty((n, V, 4), np.uint8)
    scales = np.empty(n, np.float32)
    L.check(L.load().mbir_get_sysmatrix_columns(h, vox.ctypes.data, n, first.ctypes.data,
                                                count.ctypes.data, vals.ctypes.data,
                                                codes.ctypes.data, scales.ctypes.data), h,
            "mbir_get_sysmatrix_columns")
    return first, count, vals, codes, scales


def mbir_probe_update(h, voxels):
    vox = np.ascontiguousarray(voxels, np.int64)
    n = vox.size
    t1 = np.empty(n, np.float32)
    t2 = np.empty(n, np.float32)
    dl = np.empty(n, np.float32)
    L.check(L.load().mbir_probe_update(h, vox.ctypes.data, n, t1.ctypes.data, t2.ctypes.data,
                                       dl.ctypes.data), h, "mbir_probe_update")
    return t1, t2, dl


def mbir_link_slabs(handles):
    """Test hook: link handles of consecutive slabs on one device (include/mbir.h)."""
    arr = (C.c_void_p * len(handles))(*[h.value if isinstance(h, C.c_void_p) else h for h in handles])
    L.check(L.load().mbir_link_slabs(arr, len(handles)), None, "mbir_link_slabs")


def mbir_set_update_dump(h, capacity: int):
    L.check(L.load().mbir_set_update_dump(h, int(capacity)), h, "mbir_set_update_dump")


DUMP_SAME_STATE = 1 << 62  # MBIR_DUMP_SAME_STATE: computed from the same state as the previous record


def mbir_get_update_dump(h, cap: int):
    """Returns (voxels int64 (| DUMP_SAME_STATE for a pair's second update), theta1, theta2,
    delta float32, n_recorded)."""
    vox = np.empty(cap, np.int64)
    t1 = np.empty(cap, np.float32)
    t2 = np.empty(cap, np.float32)
    dl = np.empty(cap, np.float32)
    n = C.c_int64()
    L.check(L.load().mbir_get_update_dump(h, cap, vox.ctypes.data, t1.ctypes.data, t2.ctypes.data,
                                          dl.ctypes.data, C.byref(n)), h, "mbir_get_update_dump")
    m = min(n.value, cap)
    return vox[:m], t1[:m], t2[:m], dl[:m], n.value


def mbir_get_schedule(h, g: Geometry, sizes: dict):
    """(task_list [nz][4][max_group] int32, task_count [nz][4] int32, amount [nz][nsv] float32)."""
    tl = np.empty((g.nz_local, 4, sizes["max_group"]), np.int32)
    tc = np.empty((g.nz_local, 4), np.int32)
    am = np.empty((g.nz_local, sizes["nsv"]), np.float32)
    L.check(L.load().mbir_get_schedule(h, tl.ctypes.data, tc.ctypes.data, am.ctypes.data), h,
            "mbir_get_schedule")
    return tl, tc, am


def mbir_destroy(h):
    if h:
        L.load().mbir_destroy(h)


class Reconstructor:
    """Owning wrapper around one mbir_handle."""

    def __init__(self, g: Geometry, p: Prior | None = None, o: Options | None = None, **dist):
        self.g, self.p, self.o = g, p or Prior(), o or Options()
        self.h = mbir_create(g, self.p, self.o, **dist)

    def close(self):
        if self.h:
            mbir_destroy(self.h)
            self.h = None

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def set_sinogram(self, y, w):
        mbir_set_sinogram(self.h, self.g, y, w)

    def set_image(self, x0=None):
        mbir_set_image(self.h, self.g, x0)

    def init_fbp(self):
        """x0 = FBP of the loaded sinogram (mbir_init_fbp)."""
        mbir_init_fbp(self.h)

    def reconstruct(self, equits: float) -> dict:
        return mbir_reconstruct(self.h, equits)

    def iterate(self, n: int) -> dict:
        return mbir_iterate(self.h, n)

    def image(self, out=None):
        return mbir_get_image(self.h, self.g, out)

    def error_sinogram(self, out=None):
        return mbir_get_error_sinogram(self.h, self.g, out)

    def rmse_hu(self, golden, mu_water: float = 0.02) -> float:
        return mbir_rmse_hu(self.h, self.g, golden, mu_water)

    def sizes(self) -> dict:
        return mbir_query_sizes(self.h)

    def sysmatrix(self):
        return mbir_get_sysmatrix(self.h, self.g)

    def sysmatrix_columns(self, voxels):
        return mbir_get_sysmatrix_columns(self.h, self.g, voxels)

    def probe(self, voxels):
        return mbir_probe_update(self.h, voxels)

    def set_update_dump(self, capacity: int):
        mbir_set_update_dump(self.h, capacity)

    def update_dump(self, cap: int):
        return mbir_get_update_dump(self.h, cap)

    def schedule(self):
        return mbir_get_schedule(self.h, self.g, self.sizes())
