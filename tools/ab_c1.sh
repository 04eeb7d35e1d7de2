# C1 (AlexNet, 16 images) A/B over LR environment switches: step time and LR share
cd "$GRAFT_REPO_ROOT"
for cfg in "" "VISTA_LR_FUSED=0" "VISTA_LR_DOT=0" "VISTA_LR_DOT=0 VISTA_LR_FUSED=0" "VISTA_LR_COOP=0"; do
  echo "== ${cfg:-default}"
  env $cfg timeout 300 python bench.py --config alexnet_c1 --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline $1 2>&1 | python -c "
import json,sys
for l in sys.stdin:
    if l.startswith('{'):
        d=json.loads(l); b=d['breakdown_ms']
        print('ms/step %.3f' % d['ms_per_step'], 'lr %.3f n %d' % (b['lr_pass']['ms'], b['lr_pass']['launches']), 'conv %.3f' % b['conv_fc_tcgen05']['ms'], 'launches', d['gpu_launches'])
"
done
