#!/bin/bash
# A/B timing: the in-tree library against tools/alt/$1 (outputs under gpurun_out/ab_$1.log)
B=${1:-libmbir_r1.so}; IT=${2:-6}
for r in 1 2; do
  echo "== in-tree" >> gpurun_out/ab_$B.log; timeout 200 python tools/iter_profile.py --iters $IT 2>&1 | grep "^iter" >> gpurun_out/ab_$B.log
  echo "== $B" >> gpurun_out/ab_$B.log; MBIR_LIB=tools/alt/$B timeout 200 python tools/iter_profile.py --iters $IT 2>&1 | grep "^iter" >> gpurun_out/ab_$B.log
done
