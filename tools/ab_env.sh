# bench A/B over environment settings: bash tools/ab_env.sh "ENV1=a" "ENV2=b" ...  ("" = defaults)
cd "$GRAFT_REPO_ROOT"
for cfg in "$@"; do
  echo "== ${cfg:-default}"
  env $cfg timeout 300 python bench.py --steps 8 --warmup 3 --e2e-steps 0 --no-cpu-baseline 2>&1 | python -c "
import json,sys
for l in sys.stdin:
    if l.startswith('{'):
        d=json.loads(l); b=d['breakdown_ms']
        print('ms/step %.2f' % d['ms_per_step'], 'min %.2f' % min(d['step_ms']['device']), 'conv %.2f' % b['conv_fc_tcgen05']['ms'], 'frac %.4f' % d['roofline']['frac'], 'lr %.2f' % b['lr_pass']['ms'], 'clk', d['clocks']['sm_mhz'])
"
done
