# A/B: per-layer CUDA-event tables of one bench step under different env settings
# usage: bash tools/ab_bench.sh "NAME1:ENV1=..,ENV2=.." "NAME2:..." ...
mkdir -p gpurun_out/ab
for spec in "$@"; do
  name=${spec%%:*}; envs=${spec#*:}
  env $(echo $envs | tr ',' ' ') VISTA_PROF_LOG=gpurun_out/ab/$name.tsv timeout 300 python bench.py --steps 3 --warmup 3 --e2e-steps 1 --no-cpu-baseline > gpurun_out/ab/$name.log 2>&1
  python tools/prof_table.py gpurun_out/ab/$name.tsv 40 > gpurun_out/ab/$name.txt
  echo "== $name ($envs)"; tail -1 gpurun_out/ab/$name.log | cut -c1-190; head -30 gpurun_out/ab/$name.txt
done
