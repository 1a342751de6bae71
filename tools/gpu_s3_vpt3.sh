#!/bin/bash
# (1) the cfg4 oracle golden and the side-11/13 config-5 supplement's oracle goldens on the box's
# host cores (background; oracle + synth only), (2) A/B of 8 view warps x 3 views/lane
# (tools/alt/libmbir_vpt3.so) against the in-tree 6 x 4 kernel, (3) the supplement's GPU sweep
J=$(nproc); echo "nproc $J" > gpurun_out/s3v_nproc.txt
GT=$(( J / 2 < 32 ? J / 2 : 32 )); [ $GT -lt 1 ] && GT=1
SJ=$(( J - GT )); [ $SJ -lt 1 ] && SJ=1
(timeout 2700 python tools/make_golden.py --config cfg4 --equits 60 --threads $GT --out gpurun_out/golden_cfg4.npz > gpurun_out/s3v_golden.log 2>&1 &)
(timeout 2700 python tools/sweep_goldens.py --set large --cases all --jobs $SJ > gpurun_out/s3v_sweepL_goldens.log 2>&1; echo done >> gpurun_out/s3v_sweepL_goldens.log) &
for r in 1 2; do
  echo "== in-tree" >> gpurun_out/s3v_ab.log; timeout 200 python tools/iter_profile.py --iters 6 2>&1 | grep "^iter\|nsv" >> gpurun_out/s3v_ab.log
  echo "== vpt3" >> gpurun_out/s3v_ab.log; MBIR_LIB=tools/alt/libmbir_vpt3.so timeout 200 python tools/iter_profile.py --iters 6 2>&1 | grep "^iter\|nsv" >> gpurun_out/s3v_ab.log
done
MBIR_LIB=tools/alt/libmbir_vpt3.so MBIR_PHASE_PROFILE=1 timeout 200 python tools/iter_profile.py --iters 3 > gpurun_out/s3v_phase_vpt3.log 2>&1
MBIR_LIB=tools/alt/libmbir_vpt3.so timeout 900 python -m pytest tests/test_gpu_hooks.py -q -x -p no:cacheprovider -k "every_update" > gpurun_out/s3v_hooks_vpt3.log 2>&1
for i in $(seq 1 240); do grep -q done gpurun_out/s3v_sweepL_goldens.log 2>/dev/null && break; sleep 10; done
cp goldens/sweep/oracle.jsonl gpurun_out/s3v_sweepL_oracle.jsonl 2>/dev/null
timeout 1200 python tools/sweep.py --set large --out gpurun_out/s3v_sweepL.json > gpurun_out/s3v_sweepL.log 2>&1
for i in $(seq 1 240); do grep -q '"config"' gpurun_out/s3v_golden.log 2>/dev/null && break; sleep 10; done
tail -2 gpurun_out/s3v_golden.log
