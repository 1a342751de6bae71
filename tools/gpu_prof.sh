#!/bin/bash
# A/B of the update kernel against another build (tools/alt/libmbir_r1.so) and one ncu --set full
# capture of a dense-sweep launch of the current kernel (outputs under gpurun_out/).
for r in 1 2; do
  echo "== current" >> gpurun_out/p_ab.log; timeout 200 python tools/iter_profile.py --iters 6 2>&1 | grep "^iter" >> gpurun_out/p_ab.log
  echo "== r1 kernel" >> gpurun_out/p_ab.log; MBIR_LIB=tools/alt/libmbir_r1.so timeout 200 python tools/iter_profile.py --iters 6 2>&1 | grep "^iter" >> gpurun_out/p_ab.log
done
timeout 900 ncu --set full --import-source on --clock-control none -k regex:k_svicd -s 2 -c 1 -o gpurun_out/p_svicd python tools/iter_profile.py --iters 1 > gpurun_out/p_ncu.log 2>&1
cp paper_conf_ppopp_sabnewkbrm17_b200/csrc/svicd.sm_100a.cubin gpurun_out/ 2>/dev/null
