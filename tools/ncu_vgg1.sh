# --set full capture of VGG16 conv1_1 (Cin 8 gather-row conv, 227x227) at a 1024-image micro-batch
mkdir -p gpurun_out/ncu4
ncu --set full --clock-control none --import-source on -k regex:conv_tc -s 0 -c 1 -o gpurun_out/ncu4/vgg1 \
    python bench.py --config vgg16_fc678_amazon --images 1024 --steps 1 --warmup 0 --e2e-steps 0 --no-cpu-baseline > gpurun_out/ncu4/vgg1.log 2>&1
ls -la gpurun_out/ncu4
