#!/bin/bash
for b in 42 84 126 203; do
  timeout 300 python tools/converge.py --config cfg3 --init fbp --batch-svs $b --iters 150 >> gpurun_out/conv3.jsonl 2>> gpurun_out/conv3.err
done
