# --set full captures of the ResNet stem kernel and one LR gradient pass (bench workload at 1024 images)
mkdir -p gpurun_out/ncu2
ARGS="--images 4096 --steps 1 --warmup 0 --e2e-steps 0 --no-cpu-baseline"
ncu --set full --clock-control none --import-source on -k regex:conv1_pool -s 1 -c 1 -o gpurun_out/ncu2/stem \
    python bench.py $ARGS > gpurun_out/ncu2/stem.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:lr_stream_kernel -s 30 -c 1 -o gpurun_out/ncu2/lr \
    python bench.py $ARGS > gpurun_out/ncu2/lr.log 2>&1
ls -la gpurun_out/ncu2
