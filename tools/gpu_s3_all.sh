#!/bin/bash
# One box, in order: the side-11/13 config-5 supplement (oracle goldens on 4 host cores in the
# background, then its GPU sweep), the cfg4 oracle golden on 12 host threads (oracle + synth only),
# then the session's measurement set (tools/gpu_s3_final.sh) with that golden in place.
(timeout 2400 python tools/sweep_goldens.py --set large --cases all --jobs 4 > gpurun_out/s3a_sweepL_goldens.log 2>&1; \
 cp goldens/sweep/oracle.jsonl gpurun_out/s3a_sweepL_oracle.jsonl; \
 timeout 1200 python tools/sweep.py --set large --out gpurun_out/s3a_sweepL.json > gpurun_out/s3a_sweepL.log 2>&1; \
 echo done >> gpurun_out/s3a_sweepL.log) &
SW=$!
timeout 3000 python tools/make_golden.py --config cfg4 --equits 60 --threads 12 --out gpurun_out/golden_cfg4.npz > gpurun_out/s3a_golden.log 2>&1
mkdir -p goldens && cp gpurun_out/golden_cfg4.npz goldens/golden_cfg4.npz
wait $SW
bash tools/gpu_s3_final.sh
