#!/usr/bin/env bash
# BASELINE.json configs on one B200 (per-GPU shares for the multi-GPU configs); one JSON line each.
set -u
OUT=${1:-gpurun_out/configs}
mkdir -p "$OUT"
run() { name=$1; shift; timeout 1500 python bench.py --no-cpu-baseline "$@" > "$OUT/$name.log" 2>&1; tail -1 "$OUT/$name.log" | cut -c1-220; }
run c1_alexnet            --config alexnet_c1 --steps 5 --warmup 3 --e2e-steps 2
run c2_resnet_foods20k    --steps 5 --warmup 3 --e2e-steps 2
run c3_vgg16_amazon200k   --config vgg16_fc678_amazon --steps 2 --warmup 1 --e2e-steps 1
run c4_resnet200k_staged  --config resnet50_top5_amazon200k --steps 2 --warmup 1 --e2e-steps 1 --plan staged
run c4_resnet200k_eager   --config resnet50_top5_amazon200k --steps 2 --warmup 1 --e2e-steps 1 --plan eager
run c4_resnet200k_lazy    --config resnet50_top5_amazon200k --steps 1 --warmup 1 --e2e-steps 1 --plan lazy
run c5_resnet1M_per_gpu   --config resnet50_top5_amazon200k --images 125000 --steps 2 --warmup 1 --e2e-steps 1
