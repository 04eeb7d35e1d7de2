# Round-end evidence on one B200: bench (default), reference arm, MLP/base variants, ncu launch list +
# conv DRAM traffic + one full capture, per-layer CUDA-event table, BASELINE configs.
set -u
OUT=gpurun_out/final
mkdir -p $OUT
timeout 600 python bench.py > $OUT/bench.log 2>&1
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > $OUT/bench_ref.log 2>&1
VISTA_PROF_LOG=$OUT/prof.tsv timeout 300 python bench.py --steps 1 --warmup 1 --e2e-steps 1 --no-cpu-baseline > $OUT/prof_bench.log 2>&1
python tools/prof_table.py $OUT/prof.tsv 60 > $OUT/layer_table.txt
timeout 1200 bash tools/profile_gpu.sh $OUT/ncu
timeout 2400 bash tools/run_configs.sh $OUT/configs
tail -1 $OUT/bench.log | cut -c1-300
