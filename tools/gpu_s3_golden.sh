#!/bin/bash
# The cfg4 oracle golden on all host cores (oracle + synth only, tools/make_golden.py), then the
# default bench line with it in place (cfg4 time to 10 HU against the oracle golden).
timeout 3000 python tools/make_golden.py --config cfg4 --equits 60 --threads $(nproc) --out gpurun_out/golden_cfg4.npz > gpurun_out/s3g_golden.log 2>&1
mkdir -p goldens && cp gpurun_out/golden_cfg4.npz goldens/golden_cfg4.npz && \
timeout 900 python bench.py --no-psv > gpurun_out/s3g_bench.json 2> gpurun_out/s3g_bench.err
