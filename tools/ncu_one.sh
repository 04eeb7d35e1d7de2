# --set full of one kernel launch of the bench step (CSV exports only): bash tools/ncu_one.sh NAME REGEX [SKIP] [bench args]
cd "$GRAFT_REPO_ROOT"
NAME=$1; RX=$2; SKIP=${3:-2}; shift 3
mkdir -p gpurun_out/ncu_one
timeout 600 ncu --set full --clock-control none --import-source on --kernel-name-base demangled \
    -k "regex:$RX" -s $SKIP -c 1 -o gpurun_out/ncu_one/$NAME \
    python bench.py --steps 1 --warmup 0 --e2e-steps 0 --no-cpu-baseline --images 3072 "$@" > gpurun_out/ncu_one/$NAME.log 2>&1
ncu -i gpurun_out/ncu_one/$NAME.ncu-rep --page details --csv > gpurun_out/ncu_one/$NAME.csv 2>/dev/null
ncu -i gpurun_out/ncu_one/$NAME.ncu-rep --page raw --csv > gpurun_out/ncu_one/$NAME.raw.csv 2>/dev/null
ncu -i gpurun_out/ncu_one/$NAME.ncu-rep --page source --csv --print-source sass > gpurun_out/ncu_one/$NAME.src.csv 2>/dev/null
rm -f gpurun_out/ncu_one/$NAME.ncu-rep
