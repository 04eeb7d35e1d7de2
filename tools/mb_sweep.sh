# stage-1 micro-batch sweep (bench --micro-batch): ResNet50 C2 and VGG16 C3
cd "$GRAFT_REPO_ROOT"
show() { python -c "
import json,sys
for l in open('gpurun_out/mb.json'):
    if l.startswith('{'):
        d=json.loads(l); b=d['breakdown_ms']
        print('$1 mb $2', 'ms/step %.2f' % d['ms_per_step'], 'conv %.2f' % b['conv_fc_tcgen05']['ms'], 'frac %.4f' % d['roofline']['frac'], 'clk', d['clocks']['sm_mhz'], 'peak', d['config'].get('peak_bytes',{}).get('pred') if isinstance(d['config'].get('peak_bytes'),dict) else None)
"; }
for mb in 2048 4096 1024 2048 4096; do
  timeout 300 python bench.py --steps 4 --warmup 3 --e2e-steps 0 --no-cpu-baseline --micro-batch $mb > gpurun_out/mb.json 2>&1; show c2 $mb
done
for mb in 1024 2048; do
  timeout 600 python bench.py --config vgg16_fc678_amazon --images 40000 --steps 2 --warmup 1 --e2e-steps 0 --no-cpu-baseline --micro-batch $mb > gpurun_out/mb.json 2>&1; show c3 $mb
done
