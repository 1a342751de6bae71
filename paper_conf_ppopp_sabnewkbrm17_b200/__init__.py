"""B200-native GPU-ICD (Sabne et al., PPoPP'17): SuperVoxel ICD for model-based CT
reconstruction, as a C-ABI library (libmbir.so, sm_100a) with a thin Python binding.

See include/mbir.h for the contract and DESIGN.md for the design.  Building:
``python -c "import __graft_entry__ as g; g.build()"`` (or ``make -C csrc``).
"""
from .api import (  # noqa: F401
    DUMP_SAME_STATE,
    Geometry,
    Options,
    Prior,
    Reconstructor,
    mbir_create,
    mbir_destroy,
    mbir_get_error_sinogram,
    mbir_get_image,
    mbir_get_sysmatrix,
    mbir_get_sysmatrix_columns,
    mbir_iterate,
    mbir_link_slabs,
    mbir_get_update_dump,
    mbir_set_update_dump,
    mbir_get_schedule,
    mbir_nccl_unique_id,
    mbir_probe_update,
    mbir_query_sizes,
    mbir_reconstruct,
    mbir_rmse_hu,
    mbir_set_image,
    mbir_init_fbp,
    mbir_set_sinogram,
)
from ._lib import LIB_PATH, MbirError, load  # noqa: F401
