# --set full capture of one LR power pass (CH = 2: a conv5_x layer, ld 8328, 16k train rows) and one
# gradient pass at the bench workload, source-level
cd "$GRAFT_REPO_ROOT"
mkdir -p gpurun_out/ncu_lr
ncu --set full --clock-control none --import-source on --kernel-name-base demangled \
    -k "regex:lr_stream_kernel<\(int\)2, \(int\)[23]" -s 30 -c 2 -o gpurun_out/ncu_lr/lr \
    python bench.py --steps 1 --warmup 0 --e2e-steps 0 --no-cpu-baseline > gpurun_out/ncu_lr/lr.log 2>&1
ncu -i gpurun_out/ncu_lr/lr.ncu-rep --page details --csv > gpurun_out/ncu_lr/details.csv 2>/dev/null
ncu -i gpurun_out/ncu_lr/lr.ncu-rep --page source --csv --print-source sass > gpurun_out/ncu_lr/source.csv 2>/dev/null
ls -la gpurun_out/ncu_lr
