cd "$GRAFT_REPO_ROOT"
timeout 300 python -m pytest tests/test_gpu_e2e.py -q -x -k "stem" 2>&1 | tail -2
for e in "VISTA_LR_BATCH=0" ""; do
  env $e timeout 600 python bench.py --no-cpu-baseline --config vgg16_fc678_amazon --steps 1 --warmup 1 --e2e-steps 0 > gpurun_out/c3.log 2>&1
  echo "== C3 $e $(grep -o '"peak_bytes": {[^}]*}' gpurun_out/c3.log)"
done
mkdir -p gpurun_out/p6; VISTA_PROF_LOG=gpurun_out/p6/prof.tsv timeout 300 python bench.py --steps 1 --warmup 3 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1; python tools/prof_table.py gpurun_out/p6/prof.tsv 60 | grep -E "conv1|LR|total"
bash tools/ab_env.sh "" "VISTA_LR_SHARE=1.5,4,9,9,9" "VISTA_LR_SHARE=2,4,9,9,9" "" 
