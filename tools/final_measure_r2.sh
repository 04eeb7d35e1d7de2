# Round-2 evidence on one B200: bench (default), reference arm, ncu launch list of the bench command,
# per-launch DRAM bytes of the conv class, one --set full capture of the top conv kernel (CSV exports only),
# the per-layer CUDA-event table, and the BASELINE configs.
set -u
cd "$GRAFT_REPO_ROOT"
OUT=gpurun_out/r2final
mkdir -p $OUT
timeout 600 python bench.py > $OUT/bench.log 2>&1
timeout 900 python bench.py --impl reference --steps 3 --warmup 3 > $OUT/bench_ref.log 2>&1
VISTA_PROF_LOG=$OUT/prof.tsv timeout 300 python bench.py --steps 1 --warmup 3 --e2e-steps 1 --no-cpu-baseline > $OUT/prof_bench.log 2>&1
python tools/prof_table.py $OUT/prof.tsv 60 > $OUT/layer_table.txt
ARGS="--steps 1 --warmup 0 --e2e-steps 0 --no-cpu-baseline"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches.csv \
    python bench.py $ARGS > $OUT/ncu_launches.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none \
    -k regex:"conv_tc|res_chain|conv1_pool" --csv --log-file $OUT/conv_dram.csv python bench.py $ARGS > $OUT/ncu_dram.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k regex:"conv_tc_kernel<\(int\)256, \(int\)4" -s 4 -c 1 \
    -o $OUT/conv_full python bench.py --images 3072 $ARGS > $OUT/ncu_full.log 2>&1
ncu -i $OUT/conv_full.ncu-rep --page raw --csv > $OUT/conv_full.raw.csv 2>/dev/null
ncu -i $OUT/conv_full.ncu-rep --page details --csv > $OUT/conv_full.details.csv 2>/dev/null
rm -f $OUT/conv_full.ncu-rep
timeout 2400 bash tools/run_configs.sh $OUT/configs
tail -1 $OUT/bench.log | cut -c1-300
du -sh gpurun_out
