# timing of the update kernel under development switches (MBIR_DBG bits), iteration by iteration
for d in ${DBGS:-0}; do
  echo "== dbg $d"; MBIR_DBG=$d timeout 100 python tools/iter_profile.py --iters ${ITERS:-4} ${EXTRA} 2>&1 | grep "^iter"
done
