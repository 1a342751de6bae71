#!/bin/bash
# Final check of the session: GPU tests (FBP now filters into e) and the default bench line with the
# cfg4 oracle golden in place and every CPU leg (oracle cpu_baseline, PSV-ICD).
timeout 1500 python -m pytest tests -q -m gpu -p no:cacheprovider -rf > gpurun_out/s3l_pytest_gpu.log 2>&1; echo "rc=$?" >> gpurun_out/s3l_pytest_gpu.log
timeout 1500 python bench.py > gpurun_out/s3l_bench.json 2> gpurun_out/s3l_bench.err
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/s3l_smoke.log 2>&1
