# --set full capture of the lean LR dot kernel (power pass, conv5_x layer and conv4_6 layer) at the bench workload
cd "$GRAFT_REPO_ROOT"
mkdir -p gpurun_out/ncu_lr2
ncu --set full --clock-control none --import-source on --kernel-name-base demangled \
    -k "regex:lr_dot_kernel<\(int\)[48], \(int\)[12], \(int\)2" -s 40 -c 2 -o gpurun_out/ncu_lr2/lr \
    python bench.py --steps 1 --warmup 0 --e2e-steps 0 --no-cpu-baseline > gpurun_out/ncu_lr2/lr.log 2>&1
ncu -i gpurun_out/ncu_lr2/lr.ncu-rep --page details --csv > gpurun_out/ncu_lr2/details.csv 2>/dev/null
ncu -i gpurun_out/ncu_lr2/lr.ncu-rep --page source --csv --print-source sass > gpurun_out/ncu_lr2/source.csv 2>/dev/null
ls -la gpurun_out/ncu_lr2
