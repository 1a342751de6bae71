#!/bin/bash
timeout 300 python tools/converge.py --config cfg3 --init fbp --det 1 --zero-skip 0 --iters 40 >> gpurun_out/conv2.jsonl 2>> gpurun_out/conv2.err
timeout 300 python tools/converge.py --config cfg3 --init fbp --zero-skip 0 --iters 40 >> gpurun_out/conv2.jsonl 2>> gpurun_out/conv2.err
timeout 300 python tools/converge.py --config cfg3 --init fbp --batch-svs 8 --iters 40 >> gpurun_out/conv2.jsonl 2>> gpurun_out/conv2.err
