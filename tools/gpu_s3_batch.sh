#!/bin/bash
# In-kernel batches (one cooperative launch per phase, grid barriers between batches) and the
# padded odd-warp cluster: GPU tests, cfg3/cfg4 per-iteration timing, the cfg3 bench line, and the
# side-11/13 config-5 supplement (oracle goldens on the host cores, kept under gpurun_out/).
timeout 1500 python -m pytest tests -q -m gpu -p no:cacheprovider -rf > gpurun_out/s3b_pytest_gpu.log 2>&1; echo "rc=$?" >> gpurun_out/s3b_pytest_gpu.log
(timeout 1800 python tools/sweep_goldens.py --set large --cases all --jobs 12 > gpurun_out/s3b_sweepL_goldens.log 2>&1; echo done >> gpurun_out/s3b_sweepL_goldens.log) &
SW=$!
timeout 300 python tools/iter_profile.py --config cfg3 --iters 8 > gpurun_out/s3b_iter_cfg3.log 2>&1
timeout 300 python tools/iter_profile.py --iters 6 > gpurun_out/s3b_iter_cfg4.log 2>&1
wait $SW
timeout 900 python bench.py --config cfg3 --no-cpu > gpurun_out/s3b_bench_cfg3.json 2> gpurun_out/s3b_bench_cfg3.err
mkdir -p gpurun_out/sweepL && cp goldens/sweep/sweepL*.npz goldens/sweep/oracle.jsonl gpurun_out/sweepL/ 2>/dev/null
timeout 1200 python tools/sweep.py --set large --out gpurun_out/s3b_sweepL.json > gpurun_out/s3b_sweepL.log 2>&1
