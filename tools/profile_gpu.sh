#!/usr/bin/env bash
# Collects the ncu evidence for bench.py's dominant kernel (run under gpurun, one GPU).
#  1. launch list of one bench step: every kernel with its device time (cold-cache, serialised)
#  2. dram bytes + time for every conv_tc_kernel launch of one step (traffic per launch)
#  3. one --set full capture of the largest conv launch class (source-level stalls)
set -u
OUT=${1:-gpurun_out}
mkdir -p "$OUT"
ARGS="--steps 1 --warmup 0 --e2e-steps 1 --no-cpu-baseline"
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file "$OUT/launches.csv" \
    python bench.py $ARGS > "$OUT/ncu_launches.log" 2>&1
ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none \
    -k regex:conv_tc --csv --log-file "$OUT/conv_dram.csv" python bench.py $ARGS > "$OUT/ncu_dram.log" 2>&1
ncu --set full --clock-control none --import-source on -k regex:conv_tc -s 4 -c 1 -o "$OUT/conv_full" \
    python bench.py --images 1024 $ARGS > "$OUT/ncu_full.log" 2>&1
ls -la "$OUT"
