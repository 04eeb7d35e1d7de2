# LR A/B on the bench workload: r1 kernels (unfused, VISTA_LR_DOT=0 VISTA_LR_FUSED=0), lean dot kernel
# unfused, lean dot kernel fused (default)
cd "$GRAFT_REPO_ROOT"
for cfg in ${LR_AB_CFGS:-"VISTA_LR_DOT=0 VISTA_LR_FUSED=0" "VISTA_LR_FUSED=0" ""}; do
  echo "== $cfg"
  env $cfg timeout 300 python bench.py --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline 2>&1 | python -c "
import json,sys
for l in sys.stdin:
    if l.startswith('{'):
        d=json.loads(l); b=d['breakdown_ms']
        print('ms/step', round(d['ms_per_step'],2), 'lr_pass', b.get('lr_pass'), 'lr_small', b.get('lr_small'), 'acc', d['test_acc_per_layer'])
"
done
