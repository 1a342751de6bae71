# DRAM / L2 bytes of the update kernel over ONE bench step (all its k_svicd launches), for
# bench.py's roofline `traffic` (profiles/icd_traffic.json, written by tools/traffic_json.py)
OUT=${1:-gpurun_out/traffic}
ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,lts__t_bytes.sum --clock-control none \
    -k regex:k_svicd --csv --log-file $OUT.csv \
    python bench.py --steps 1 --warmup 0 --no-e2e --no-converge --no-cpu > $OUT.json 2> $OUT.err
