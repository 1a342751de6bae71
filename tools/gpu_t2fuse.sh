#!/bin/bash
# fused theta2 pass: hook/replay tests, A/B against the previous library, then the GPU suite
timeout 300 python -m pytest tests/test_gpu_hooks.py -x -q -s > gpurun_out/t2_hooks.log 2>&1; echo "hooks rc=$?" >> gpurun_out/t2_hooks.log
for r in 1 2; do
  echo "== in-tree" >> gpurun_out/t2_ab.log; timeout 200 python tools/iter_profile.py --iters 6 2>&1 | grep -E "^iter|^first|^set_" >> gpurun_out/t2_ab.log
  echo "== prev" >> gpurun_out/t2_ab.log; MBIR_LIB=tools/alt/libmbir_prev.so timeout 200 python tools/iter_profile.py --iters 6 2>&1 | grep -E "^iter|^first|^set_" >> gpurun_out/t2_ab.log
done
timeout 900 python -m pytest tests -q -m gpu -x -p no:cacheprovider > gpurun_out/t2_pytest_gpu.log 2>&1; echo "gpu rc=$?" >> gpurun_out/t2_pytest_gpu.log
