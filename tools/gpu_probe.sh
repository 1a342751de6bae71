#!/bin/bash
# One GPU call's diagnostic set (outputs under gpurun_out/): host description, the GPU tests, and
# per-iteration timings of cfg4 (with the phase profile) and cfg3.
nproc > gpurun_out/box.txt; lscpu | head -20 >> gpurun_out/box.txt; nvidia-smi >> gpurun_out/box.txt
timeout 600 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1
MBIR_PHASE_PROFILE=1 timeout 300 python tools/iter_profile.py --iters 12 > gpurun_out/iter_cfg4.log 2>&1
timeout 300 python tools/iter_profile.py --config cfg3 --iters 12 > gpurun_out/iter_cfg3.log 2>&1
