#!/bin/bash
# phase profile (cycles per visit: order / pack / voxel loop / write-back) on cfg4 and cfg3, and one
# ncu --set full capture of a dense update-kernel launch (outputs under gpurun_out/)
MBIR_PHASE_PROFILE=1 timeout 300 python tools/iter_profile.py --iters 6 > gpurun_out/s3_phase_cfg4.log 2>&1
MBIR_PHASE_PROFILE=1 timeout 300 python tools/iter_profile.py --config cfg3 --iters 6 > gpurun_out/s3_phase_cfg3.log 2>&1
timeout 900 ncu --set full --import-source on --clock-control none -k regex:k_svicd -s 2 -c 1 -o gpurun_out/s3_svicd python tools/iter_profile.py --iters 3 > gpurun_out/s3_ncu.log 2>&1
python tools/ncu_summary.py gpurun_out/s3_svicd.ncu-rep 60 > gpurun_out/s3_ncu_summary.txt 2>&1
