# --set full of the res3 3x3 halo conv (one launch at the bench's micro-batch) as the CTA pair
# (VISTA_CG2=1) and as the multicast pair (VISTA_CG2=0); CSV exports only
cd "$GRAFT_REPO_ROOT"
mkdir -p gpurun_out/ncu_cg2
for c in 0 1; do
  VISTA_CG2=$c timeout 600 ncu --set full --clock-control none --import-source on --kernel-name-base demangled \
      -k "regex:conv_tc_kernel<\(int\)128, \(int\)7" -s 2 -c 1 -o gpurun_out/ncu_cg2/k$c \
      python bench.py --steps 1 --warmup 0 --e2e-steps 0 --no-cpu-baseline --images 3072 > gpurun_out/ncu_cg2/k$c.log 2>&1
  ncu -i gpurun_out/ncu_cg2/k$c.ncu-rep --page details --csv > gpurun_out/ncu_cg2/k$c.csv 2>/dev/null
  ncu -i gpurun_out/ncu_cg2/k$c.ncu-rep --page raw --csv > gpurun_out/ncu_cg2/k$c.raw.csv 2>/dev/null
  ncu -i gpurun_out/ncu_cg2/k$c.ncu-rep --page source --csv --print-source sass > gpurun_out/ncu_cg2/k$c.src.csv 2>/dev/null
  rm -f gpurun_out/ncu_cg2/k$c.ncu-rep
done
ls -la gpurun_out/ncu_cg2
