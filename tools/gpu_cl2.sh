#!/bin/bash
# cluster = 2 checks + FBP init timing (outputs under gpurun_out/)
timeout 400 python -m pytest tests/test_gpu_hooks.py -x -q -s > gpurun_out/c_hooks.log 2>&1; echo "rc=$?" >> gpurun_out/c_hooks.log
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "bench_shape or cluster" > gpurun_out/c_parity.log 2>&1; echo "rc=$?" >> gpurun_out/c_parity.log
timeout 300 python tools/fbp_time.py > gpurun_out/c_fbp.log 2>&1
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"k_(ramp|backproject|forward)" --csv --log-file gpurun_out/c_fbp_launches.csv python tools/fbp_time.py > /dev/null 2>&1
timeout 200 python tools/iter_profile.py --iters 6 --cluster 2 > gpurun_out/c_iter_cl2.log 2>&1
timeout 200 python tools/iter_profile.py --config cfg3 --iters 6 --cluster 1 > gpurun_out/c_iter_cfg3_cl1.log 2>&1
timeout 200 python tools/iter_profile.py --config cfg3 --iters 6 --cluster 2 > gpurun_out/c_iter_cfg3_cl2.log 2>&1
