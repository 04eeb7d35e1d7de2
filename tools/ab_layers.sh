# per-layer CUDA-event tables of one bench step under two environment settings: bash tools/ab_layers.sh "ENV_A" "ENV_B"
cd "$GRAFT_REPO_ROOT"
mkdir -p gpurun_out/ab_layers
i=0
for cfg in "$@"; do
  i=$((i+1))
  env $cfg VISTA_PROF_LOG=gpurun_out/ab_layers/p$i.tsv timeout 300 python bench.py --steps 1 --warmup 3 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
  python tools/prof_table.py gpurun_out/ab_layers/p$i.tsv 60 > gpurun_out/ab_layers/t$i.txt
  echo "== ${cfg:-default}"; head -16 gpurun_out/ab_layers/t$i.txt | cut -c1-150; tail -1 gpurun_out/ab_layers/t$i.txt
done
