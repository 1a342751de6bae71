#!/bin/bash
timeout 300 python -m pytest tests/test_gpu_hooks.py -x -q -s -k "every_update" > gpurun_out/t2_hooks.log 2>&1; echo "rc=$?" >> gpurun_out/t2_hooks.log
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"k_theta2" --csv --log-file gpurun_out/t2_launches.csv python tools/iter_profile.py --iters 1 > /dev/null 2>&1
