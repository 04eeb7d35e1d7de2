# A/B of two library builds in one job: bash tools/ab_lib.sh <libA.so> <libB.so>; per-layer tables + step times
cd "$GRAFT_REPO_ROOT"
mkdir -p gpurun_out/ablib
for r in 1 2; do
  for lib in "$1" "$2"; do
    tag=$(basename $lib .so)
    VISTA_LIB_PATH=$lib VISTA_PROF_LOG=gpurun_out/ablib/$tag.r$r.tsv timeout 300 python bench.py --steps 8 --warmup 3 --e2e-steps 0 --no-cpu-baseline > gpurun_out/ablib/$tag.r$r.json 2>&1
    python -c "
import json,sys
for l in open('gpurun_out/ablib/$tag.r$r.json'):
    if l.startswith('{'):
        d=json.loads(l); b=d['breakdown_ms']
        print('$tag r$r', 'ms/step %.2f' % d['ms_per_step'], 'min %.2f' % min(d['step_ms']['device']), 'conv %.2f' % b['conv_fc_tcgen05']['ms'], 'clk', d['clocks']['sm_mhz'], 'pw', d['clocks'].get('power_w_median'))
"
  done
done
for lib in "$1" "$2"; do tag=$(basename $lib .so); echo "== $tag"; python tools/prof_table.py gpurun_out/ablib/$tag.r2.tsv 24; done
