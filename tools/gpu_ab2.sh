#!/bin/bash
# A/B: in-tree library vs tools/alt/$1, cfg4 per-iteration times (gpurun_out/ab2_$1.log)
B=${1:-libmbir_prev.so}
for r in 1 2 3; do
  echo "== in-tree" >> gpurun_out/ab2_$B.log; timeout 200 python tools/iter_profile.py --iters 6 2>&1 | grep -E "^iter" >> gpurun_out/ab2_$B.log
  echo "== $B" >> gpurun_out/ab2_$B.log; MBIR_LIB=tools/alt/$B timeout 200 python tools/iter_profile.py --iters 6 2>&1 | grep -E "^iter" >> gpurun_out/ab2_$B.log
done
