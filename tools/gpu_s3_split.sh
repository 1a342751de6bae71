#!/bin/bash
# after splitting the update kernel's instantiations over four translation units: GPU tests, smoke,
# and per-iteration timing (cfg4, cfg3)
timeout 1500 python -m pytest tests -q -m gpu -p no:cacheprovider -rf > gpurun_out/s3s_pytest_gpu.log 2>&1; echo "rc=$?" >> gpurun_out/s3s_pytest_gpu.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/s3s_smoke.log 2>&1
timeout 300 python tools/iter_profile.py --iters 6 2>&1 | grep "^iter" > gpurun_out/s3s_iter_cfg4.log
timeout 300 python tools/iter_profile.py --config cfg3 --iters 6 2>&1 | grep "^iter" > gpurun_out/s3s_iter_cfg3.log
