mkdir -p gpurun_out/mb
for mb in 128 256 512; do
  VISTA_PROF_LOG=gpurun_out/mb/prof$mb.tsv timeout 300 python bench.py --steps 2 --warmup 1 --e2e-steps 1 --no-cpu-baseline --micro-batch $mb > gpurun_out/mb/b$mb.log 2>&1
  python tools/prof_table.py gpurun_out/mb/prof$mb.tsv 24 > gpurun_out/mb/t$mb.txt
  echo "== mb $mb"; tail -1 gpurun_out/mb/b$mb.log | cut -c1-200; cat gpurun_out/mb/t$mb.txt
done
