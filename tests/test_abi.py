"""CPU-side checks of the C-ABI boundary: libmbir.so loads, exports every symbol include/mbir.h
declares, and its host-only helpers behave (no compute calls without a GPU)."""
import ctypes as C
import os
import re
import subprocess

import pytest

import paper_conf_ppopp_sabnewkbrm17_b200 as M
from paper_conf_ppopp_sabnewkbrm17_b200 import _lib as L

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "mbir.h")


def declared_functions():
    src = open(HEADER).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(mbir_[a-z_0-9]+)\s*\(", src)))


def test_header_declares_the_binding_exports():
    assert sorted(L.EXPORTS) == declared_functions()


def test_library_loads_and_exports_every_symbol():
    lib = M.load()
    for name in declared_functions():
        assert hasattr(lib, name), name
    out = subprocess.run(["nm", "-D", "--defined-only", M.LIB_PATH], capture_output=True,
                         text=True, check=True).stdout
    for name in declared_functions():
        assert re.search(rf"\bT {name}\b", out), f"{name} not exported"


def test_library_is_sm100a():
    out = subprocess.run(["cuobjdump", "--list-elf", M.LIB_PATH], capture_output=True,
                         text=True).stdout
    assert "sm_100a" in out


def test_host_helpers():
    lib = M.load()
    o = L.mbir_options()
    lib.mbir_default_options(C.byref(o))
    assert (o.sv_side, o.sv_fraction, o.batch_svs, o.batch_threshold, o.zero_skip, o.quantize_A) == (
        9, 0.25, 0, -1, 1, 1)
    p = L.mbir_prior()
    lib.mbir_default_prior(C.byref(p))
    assert (p.p, p.q, p.T, p.neighborhood, p.positivity) == (1.2, 2.0, 1.0, 26, 1)
    assert lib.mbir_strerror(L.MBIR_EINVAL) == b"invalid argument"
    assert lib.mbir_strerror(12345) == b"unknown error"
    assert lib.mbir_last_error(None) == b"null handle"
    lib.mbir_destroy(None)  # NULL-safe


def test_struct_layouts_match_header():
    """ctypes mirrors of the C structs have the sizes the C compiler gives them."""
    src = f"""
#include <stdio.h>
#include "{HEADER}"
int main(void) {{
  printf("%zu %zu %zu %zu %zu %zu\\n", sizeof(mbir_geometry), sizeof(mbir_prior),
         sizeof(mbir_options), sizeof(mbir_dist), sizeof(mbir_stats), sizeof(mbir_sizes));
  return 0;
}}"""
    d = "/tmp/mbir_abi_check"
    os.makedirs(d, exist_ok=True)
    open(f"{d}/t.c", "w").write(src)
    subprocess.check_call(["gcc", "-o", f"{d}/t", f"{d}/t.c"])
    sizes = list(map(int, subprocess.check_output([f"{d}/t"]).split()))
    assert sizes == [C.sizeof(L.mbir_geometry), C.sizeof(L.mbir_prior), C.sizeof(L.mbir_options),
                     C.sizeof(L.mbir_dist), C.sizeof(L.mbir_stats), C.sizeof(L.mbir_sizes)]


def test_null_arguments_rejected_without_touching_the_gpu():
    lib = M.load()
    h = C.c_void_p()
    assert lib.mbir_create(None, None, None, None, C.byref(h)) == L.MBIR_EINVAL
    assert lib.mbir_create(None, None, None, None, None) == L.MBIR_EINVAL
    assert lib.mbir_reconstruct(None, 1.0, None) == L.MBIR_EINVAL
    assert lib.mbir_set_sinogram(None, None, None, 0) == L.MBIR_EINVAL
    assert lib.mbir_nccl_unique_id(None) == L.MBIR_EINVAL


def test_product_fails_loudly_without_library(tmp_path):
    with pytest.raises(ImportError):
        L.load.__wrapped__ if hasattr(L.load, "__wrapped__") else None
        saved = L._lib
        try:
            L._lib = None
            L.load(str(tmp_path / "missing.so"))
        finally:
            L._lib = saved
