# --set full capture of one LR power pass (CH = 3: a conv5_x layer, ld 8328) at the bench workload
mkdir -p gpurun_out/ncu3
ncu --set full --clock-control none --import-source on --kernel-name-base demangled \
    -k "regex:lr_stream_kernel<\(int\)3, \(int\)2" -s 25 -c 1 -o gpurun_out/ncu3/lr \
    python bench.py --steps 1 --warmup 0 --e2e-steps 0 --no-cpu-baseline > gpurun_out/ncu3/lr.log 2>&1
ls -la gpurun_out/ncu3
