# --set full captures (one launch each) of the conv-path kernels that matter most, at the bench's
# micro-batch (1024 images), source-level; summaries via tools/ncu_csv.py-style CSV exports
cd "$GRAFT_REPO_ROOT"
mkdir -p gpurun_out/ncu_conv
i=0
for k in "regex:conv_tc_kernel<\(int\)128, \(int\)2, \(bool\)1, \(int\)3, \(int\)4>" \
         "regex:res_chain_kernel<\(int\)128" "regex:conv1_pool_kernel" \
         "regex:conv_tc_kernel<\(int\)128, \(int\)7" "regex:conv_tc_kernel<\(int\)64, \(int\)7" \
         "regex:res_chain_kernel<\(int\)64" "regex:conv_tc_kernel<\(int\)256, \(int\)2, \(bool\)0"; do
  i=$((i+1))
  timeout 600 ncu --set full --clock-control none --import-source on --kernel-name-base demangled \
      -k "$k" -s 2 -c 1 -o gpurun_out/ncu_conv/k$i \
      python bench.py --steps 1 --warmup 0 --e2e-steps 0 --no-cpu-baseline --images 3072 > gpurun_out/ncu_conv/k$i.log 2>&1
  ncu -i gpurun_out/ncu_conv/k$i.ncu-rep --page details --csv > gpurun_out/ncu_conv/k$i.csv 2>/dev/null
  ncu -i gpurun_out/ncu_conv/k$i.ncu-rep --page raw --csv > gpurun_out/ncu_conv/k$i.raw.csv 2>/dev/null
  ncu -i gpurun_out/ncu_conv/k$i.ncu-rep --page source --csv --print-source sass > gpurun_out/ncu_conv/k$i.src.csv 2>/dev/null
  rm -f gpurun_out/ncu_conv/k$i.ncu-rep
done
ls -la gpurun_out/ncu_conv
