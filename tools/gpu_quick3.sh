#!/bin/bash
timeout 300 python -m pytest tests/test_gpu_hooks.py -x -q -s > gpurun_out/q_hooks.log 2>&1; echo "hooks rc=$?" >> gpurun_out/q_hooks.log
rm -f gpurun_out/ab_libmbir_prev.so.log; bash tools/gpu_ab.sh libmbir_prev.so 6
MBIR_PHASE_PROFILE=1 timeout 200 python tools/iter_profile.py --iters 6 > gpurun_out/q_iter_cfg4_prof.log 2>&1
timeout 900 python -m pytest tests -q -m gpu -x -p no:cacheprovider > gpurun_out/q_pytest_gpu.log 2>&1; echo "gpu rc=$?" >> gpurun_out/q_pytest_gpu.log
