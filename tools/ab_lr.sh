# LR per-pass A/B of two library builds in one job: bash tools/ab_lr.sh libA.so libB.so
cd "$GRAFT_REPO_ROOT"
mkdir -p gpurun_out/ablr
for r in 1 2; do
  for lib in "$1" "$2"; do
    tag=$(basename $lib .so)
    VISTA_LIB_PATH=$lib VISTA_PROF_LOG=gpurun_out/ablr/$tag.r$r.tsv timeout 300 python bench.py --steps 1 --warmup 3 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
    echo "== $tag r$r"; python tools/lr_passes.py gpurun_out/ablr/$tag.r$r.tsv | tail -3
    python - <<PY
rows=[l.rstrip('\n').split('\t') for l in open('gpurun_out/ablr/$tag.r$r.tsv')]
lr=[(float(r[1]),float(r[3])) for r in rows if r[0]=='5']
seq=[round(ms*1e3,1) for ms,b in lr if abs(b-267.4e6)<1e6]
print('power', sum(seq[2:22])/20, 'ista', sum(seq[22:32])/10, 'eval', seq[32])
PY
  done
done
