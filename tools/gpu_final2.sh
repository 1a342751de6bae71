#!/bin/bash
# the 200-case sweep (stage 2) and the round's measurement set (tools/final_measure.sh)
timeout 2400 python tools/sweep.py --out gpurun_out/sweep200.json > gpurun_out/sweep200.log 2>&1
bash tools/final_measure.sh
