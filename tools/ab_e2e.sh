# e2e A/B of two library builds in one job: bash tools/ab_e2e.sh libA.so libB.so
cd "$GRAFT_REPO_ROOT"
for r in 1 2; do
  for lib in "$1" "$2"; do
    VISTA_LIB_PATH=$lib timeout 400 python bench.py --steps 5 --warmup 3 --e2e-steps 5 --no-cpu-baseline 2>&1 | python -c "
import json,sys
for l in sys.stdin:
    if l.startswith('{'):
        d=json.loads(l); print('$(basename $lib .so) r$r', 'device ms %.2f' % d['ms_per_step'], 'e2e ms %.2f' % d['e2e']['ms_per_step'], 'e2e steps', d['step_ms']['e2e'])
"
  done
done
