# Per-kernel ncu evidence: tensor-pipe utilisation of every conv/FC launch and DRAM
# throughput of the tap / join / concat / LR kernels, over one bench step (4096 images; --clock-control none)
OUT=${1:-gpurun_out/evidence}
mkdir -p "$OUT"
ncu --clock-control none --csv --log-file "$OUT/evidence.csv" \
    --metrics gpu__time_duration.sum,sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed,dram__bytes_read.sum,dram__bytes_write.sum,gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed \
    python bench.py --images 4096 --steps 1 --warmup 0 --e2e-steps 0 --no-cpu-baseline > "$OUT/evidence.log" 2>&1
ls -la "$OUT"
