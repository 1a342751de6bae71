#!/bin/bash
# Session-3 measurement set on one B200 (outputs under gpurun_out/s3z_*): the GPU test suite, the
# default bench line (with the oracle cpu_baseline and the PSV-ICD leg; the cfg4 golden when
# goldens/golden_cfg4.npz is present), the cfg3 / cfg2 lines, the update kernel's ncu
# --set full capture, the bench's launch list and the update kernel's DRAM traffic per step.
# Nothing here is a bench value except the bench*.json lines.
set -x
nproc > gpurun_out/s3z_nproc.txt
# same-box A/B: the in-tree kernel (in-kernel batches) against tools/alt/libmbir_ff.so (one launch
# per batch), cfg4 and cfg3 per-iteration device time
if [ -f tools/alt/libmbir_ff.so ]; then
  for r in 1 2; do
    for c in cfg4 cfg3; do
      echo "== in-tree $c" >> gpurun_out/s3z_ab.log; timeout 200 python tools/iter_profile.py --config $c --iters 6 2>&1 | grep "^iter" >> gpurun_out/s3z_ab.log
      echo "== ff $c" >> gpurun_out/s3z_ab.log; MBIR_LIB=tools/alt/libmbir_ff.so timeout 200 python tools/iter_profile.py --config $c --iters 6 2>&1 | grep "^iter" >> gpurun_out/s3z_ab.log
    done
  done
fi
timeout 1500 python -m pytest tests -q -m gpu -p no:cacheprovider -rf > gpurun_out/s3z_pytest_gpu.log 2>&1; echo "rc=$?" >> gpurun_out/s3z_pytest_gpu.log
timeout 1500 python bench.py > gpurun_out/s3z_bench.json 2> gpurun_out/s3z_bench.err
timeout 900 python bench.py --config cfg3 --no-cpu > gpurun_out/s3z_bench_cfg3.json 2> gpurun_out/s3z_bench_cfg3.err
timeout 600 python bench.py --config cfg2 --no-cpu --no-converge > gpurun_out/s3z_bench_cfg2.json 2> gpurun_out/s3z_bench_cfg2.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"k_(svicd|select|flatten|theta2|forward|rmse|finite|columns|bands|probe|ramp|backproject|zero)" -c 4000 --csv --log-file gpurun_out/s3z_launches.csv python bench.py --steps 2 --warmup 1 --no-e2e --no-converge --no-cpu > gpurun_out/s3z_b_ncu.log 2>&1
python tools/launch_summary.py gpurun_out/s3z_launches.csv > gpurun_out/s3z_launch_summary.txt 2>&1
timeout 900 ncu --set full --import-source on --clock-control none -k regex:k_svicd -s 2 -c 1 -o gpurun_out/s3z_svicd python tools/iter_profile.py --iters 1 > gpurun_out/s3z_ncu_full.log 2>&1
python tools/ncu_summary.py gpurun_out/s3z_svicd.ncu-rep 40 > gpurun_out/s3z_ncu_summary.txt 2>&1
ncu -i gpurun_out/s3z_svicd.ncu-rep --page raw --csv > gpurun_out/s3z_svicd_raw.csv 2>/dev/null
rm -f gpurun_out/s3z_svicd.ncu-rep  # (45 MB: gpurun copies back <= 64 MiB)
timeout 900 bash tools/traffic.sh gpurun_out/s3z_traffic
