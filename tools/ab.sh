#!/bin/bash
# A/B timing of two builds of libmbir on one box: tools/ab.sh <libB> [iters] [reps]
B=$1; IT=${2:-4}; REPS=${3:-2}
for r in $(seq $REPS); do
  echo "== A (in-tree)"; timeout 200 python tools/iter_profile.py --iters $IT 2>&1 | grep "^iter"
  echo "== B ($B)"; MBIR_LIB=$B timeout 200 python tools/iter_profile.py --iters $IT 2>&1 | grep "^iter"
done
