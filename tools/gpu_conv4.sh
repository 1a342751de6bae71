#!/bin/bash
# a non-converging config-5 case (sweep152: baggage 256^2, 180 views, lambda0 1e3, side 5) under variations
for args in "--zero-skip 1" "--zero-skip 0" "--batch-svs 20" "--batch-svs 10" "--period 2" "--sv-side 7"; do
  echo "== $args" >> gpurun_out/conv4.log
  timeout 300 python tools/converge.py --sweep 152 --iters 300 $args 2>&1 | python3 -c "
import json,sys
for l in sys.stdin:
    try: d=json.loads(l)
    except Exception: print(l.strip()); continue
    c=d['curve']; print(d['to_target'], 'final', d['final_hu'], [x[1:] for x in c[::30]])" >> gpurun_out/conv4.log
done
