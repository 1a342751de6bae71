#!/bin/bash
# GPU test pass (outputs under gpurun_out/): the new hook tests verbosely, then the whole -m gpu suite.
timeout 900 python -m pytest tests/test_gpu_hooks.py -x -q -s -m gpu > gpurun_out/pytest_hooks.log 2>&1
timeout 1200 python -m pytest tests -q -m gpu -s -p no:cacheprovider > gpurun_out/pytest_gpu.log 2>&1
