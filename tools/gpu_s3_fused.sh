#!/bin/bash
# fused write-back + next pack: GPU tests, then the per-iteration phase profile and timing (cfg4, cfg3)
timeout 1500 python -m pytest tests -q -m gpu -p no:cacheprovider -x > gpurun_out/s3f_pytest_gpu.log 2>&1; echo "rc=$?" >> gpurun_out/s3f_pytest_gpu.log
MBIR_PHASE_PROFILE=1 timeout 300 python tools/iter_profile.py --iters 6 > gpurun_out/s3f_phase_cfg4.log 2>&1
MBIR_PHASE_PROFILE=1 timeout 300 python tools/iter_profile.py --config cfg3 --iters 6 > gpurun_out/s3f_phase_cfg3.log 2>&1
timeout 300 python tools/iter_profile.py --iters 6 > gpurun_out/s3f_iter_cfg4.log 2>&1
timeout 600 python bench.py --no-cpu > gpurun_out/s3f_bench.json 2> gpurun_out/s3f_bench.err
