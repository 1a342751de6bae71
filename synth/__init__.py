"""Seeded synthetic workload generator shared by the oracle tests and the CUDA-path tests/bench.

Holds none of the method's arithmetic: no system matrix, no ICD, no prior.  It draws
Shepp-Logan-style phantoms and computes their *analytic* parallel-beam line integrals
(ellipse/ellipsoid chord lengths, averaged over sub-rays per channel -- no inverse crime),
then Poisson counts.  Recipe: DESIGN.md "Input recipe".
"""
from .phantom import (  # noqa: F401
    CONFIGS,
    Case,
    WorkloadConfig,
    baggage_phantom,
    make_case,
    make_sinogram_torch,
    noisy_counts,
    slice_ellipses,
    phantom_image,
    shepp_logan_2d,
    shepp_logan_3d,
    sinogram,
    sweep_configs,
)
