# LR per-pass A/B over environment settings in one job: bash tools/lr_env_ab.sh "ENV=a" "" ...
cd "$GRAFT_REPO_ROOT"
mkdir -p gpurun_out/lrab
i=0
for cfg in "$@"; do
  i=$((i+1))
  env $cfg VISTA_PROF_LOG=gpurun_out/lrab/p$i.tsv timeout 300 python bench.py --steps 1 --warmup 3 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
  echo "== ${cfg:-default}"; python tools/lr_passes.py gpurun_out/lrab/p$i.tsv | grep -v sequence
done
