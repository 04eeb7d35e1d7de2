# one fused LR pass launch of the C1 (AlexNet, 16 images) workload under ncu --set full, CSV exports only
cd "$GRAFT_REPO_ROOT"
mkdir -p gpurun_out/ncu_lr_c1
timeout 600 ncu --set full --clock-control none --import-source on --kernel-name-base demangled \
    -k "regex:lr_dot_kernel" -s 10 -c 1 -o gpurun_out/ncu_lr_c1/k \
    python bench.py --config alexnet_c1 --steps 1 --warmup 1 --e2e-steps 0 --no-cpu-baseline > gpurun_out/ncu_lr_c1/k.log 2>&1
ncu -i gpurun_out/ncu_lr_c1/k.ncu-rep --page details --csv > gpurun_out/ncu_lr_c1/k.csv 2>/dev/null
ncu -i gpurun_out/ncu_lr_c1/k.ncu-rep --page raw --csv > gpurun_out/ncu_lr_c1/k.raw.csv 2>/dev/null
ncu -i gpurun_out/ncu_lr_c1/k.ncu-rep --page source --csv --print-source sass > gpurun_out/ncu_lr_c1/k.src.csv 2>/dev/null
rm -f gpurun_out/ncu_lr_c1/k.ncu-rep
