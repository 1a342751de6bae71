#!/bin/bash
# The round's measurement set on one B200 (outputs under gpurun_out/): the GPU test suite, the
# default bench line, the update kernel's ncu --set full capture (one dense-iteration launch), the
# bench's launch list (gpu__time_duration, clock control none) and the per-step DRAM traffic.
# Nothing here is a bench value except bench.json.
set -x
timeout 1200 python -m pytest tests -q -m gpu -p no:cacheprovider > gpurun_out/f_pytest_gpu.log 2>&1
timeout 1500 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err
timeout 900 python bench.py --config cfg3 --no-cpu > gpurun_out/bench_cfg3.json 2> gpurun_out/bench_cfg3.err
timeout 600 python bench.py --config cfg2 --no-cpu --no-converge > gpurun_out/bench_cfg2.json 2> gpurun_out/bench_cfg2.err
timeout 600 ncu --set full --import-source on --clock-control none -k regex:k_svicd -s 2 -c 1 -o gpurun_out/svicd_full python tools/iter_profile.py --iters 1 > gpurun_out/ncu_full.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"k_(svicd|select|flatten|theta2|forward|rmse|finite|columns|bands|probe|ramp|backproject|zero)" -c 4000 --csv --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 1 --no-e2e --no-converge --no-cpu > gpurun_out/b_ncu.log 2>&1
timeout 900 bash tools/traffic.sh gpurun_out/traffic
