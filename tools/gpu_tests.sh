#!/bin/bash
# the GPU test suite (outputs under gpurun_out/)
timeout 1200 python -m pytest tests -q -m gpu -p no:cacheprovider -rA 2>&1 | tail -120 > gpurun_out/t_pytest_gpu.log; echo "gpu rc=${PIPESTATUS[0]}" >> gpurun_out/t_pytest_gpu.log
