# The round's measurement set on one B200 (outputs under gpurun_out/): the default bench line, the
# update kernel's ncu --set full capture (one dense-iteration launch), the bench's launch list and
# the per-step DRAM traffic.  Nothing here is a bench value except bench.json.
set -x
timeout 600 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err
timeout 600 ncu --set full --import-source on --clock-control none -k regex:k_icd_sv -s 2 -c 1 -o gpurun_out/icd_full python tools/iter_profile.py --iters 1 > gpurun_out/ncu_full.log 2>&1
timeout 400 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"k_(icd|select|flatten|theta2|forward|rmse|finite|columns|bands|probe|ramp|backproject|zero)" -c 3000 --csv --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 1 --no-e2e --no-converge --no-cpu > gpurun_out/b_ncu.log 2>&1
bash tools/traffic.sh gpurun_out/traffic
