#!/bin/bash
# convergence runs for cfg3 (outputs gpurun_out/conv_cfg3.jsonl)
for init in fbp zero; do
  for b in 0 100000; do
    timeout 300 python tools/converge.py --config cfg3 --init $init --batch-svs $b --iters 60 >> gpurun_out/conv_cfg3.jsonl 2>> gpurun_out/conv_cfg3.err
  done
done
