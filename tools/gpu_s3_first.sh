set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 1500 python -m pytest tests -q -m gpu -p no:cacheprovider -rf -x > gpurun_out/s3_pytest_gpu.log 2>&1; echo "rc=$?" >> gpurun_out/s3_pytest_gpu.log
timeout 900 python bench.py > gpurun_out/s3_bench.json 2> gpurun_out/s3_bench.err
