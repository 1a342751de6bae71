#!/bin/bash
# large SVs (two-window bands, auto 2-CTA cluster): hook/replay + parity tests, A/B of the default
# side-9 path against the previous library, per-iteration timing at side 11 / 13 on cfg4
timeout 600 python -m pytest tests/test_gpu_hooks.py tests/test_gpu_parity.py -x -q -s -k "large or side11 or hot_kernel" -p no:cacheprovider > gpurun_out/l_tests.log 2>&1; echo "rc=$?" >> gpurun_out/l_tests.log
for r in 1 2; do
  echo "== in-tree" >> gpurun_out/l_ab.log; timeout 200 python tools/iter_profile.py --iters 6 2>&1 | grep -E "^iter" >> gpurun_out/l_ab.log
  echo "== prev" >> gpurun_out/l_ab.log; MBIR_LIB=tools/alt/libmbir_prev.so timeout 200 python tools/iter_profile.py --iters 6 2>&1 | grep -E "^iter" >> gpurun_out/l_ab.log
done
for s in 11 13; do
  echo "== side $s" >> gpurun_out/l_ab.log; timeout 300 python tools/iter_profile.py --iters 6 --sv-side $s 2>&1 | grep -E "^iter|^\{" >> gpurun_out/l_ab.log
done
timeout 900 python -m pytest tests -q -m gpu -x -p no:cacheprovider > gpurun_out/l_pytest_gpu.log 2>&1; echo "gpu rc=$?" >> gpurun_out/l_pytest_gpu.log
