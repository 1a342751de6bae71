#!/bin/bash
# voxel pairs: hook/replay tests, per-iteration timing pairs vs single, convergence, GPU suite
timeout 400 python -m pytest tests/test_gpu_hooks.py -x -q -s > gpurun_out/p_hooks.log 2>&1; echo "hooks rc=$?" >> gpurun_out/p_hooks.log
for r in 1 2; do
  for v in 2 1; do
    echo "== vps $v" >> gpurun_out/p_ab.log; timeout 200 python tools/iter_profile.py --iters 6 --vps $v 2>&1 | grep -E "^iter|^first" >> gpurun_out/p_ab.log
  done
done
echo "== cfg3 vps 2" >> gpurun_out/p_ab.log; timeout 200 python tools/iter_profile.py --config cfg3 --iters 6 --vps 2 2>&1 | grep -E "^iter" >> gpurun_out/p_ab.log
echo "== cfg3 vps 1" >> gpurun_out/p_ab.log; timeout 200 python tools/iter_profile.py --config cfg3 --iters 6 --vps 1 2>&1 | grep -E "^iter" >> gpurun_out/p_ab.log
timeout 900 python bench.py --no-e2e --no-cpu > gpurun_out/p_bench.json 2> gpurun_out/p_bench.err
timeout 900 python -m pytest tests -q -m gpu -x -p no:cacheprovider > gpurun_out/p_pytest_gpu.log 2>&1; echo "gpu rc=$?" >> gpurun_out/p_pytest_gpu.log
