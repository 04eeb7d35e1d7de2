# compute-sanitizer over the small cases of tools/sanitize_case.py; one log per (tool, case),
# summary lines collected in gpurun_out/sanitize/summary.txt
cd "$GRAFT_REPO_ROOT"
mkdir -p gpurun_out/sanitize
S=gpurun_out/sanitize
: > $S/summary.txt
for tool in memcheck racecheck synccheck initcheck; do
  for case in resnet resnet_mc alexnet vgg lr_unfused mlp; do
    if [ "$tool" = "racecheck" ] && [ "$case" = "resnet_mc" ]; then continue; fi
    timeout 900 compute-sanitizer --tool $tool --error-exitcode 99 --print-limit 20 \
        python tools/sanitize_case.py $case > $S/$tool.$case.log 2>&1
    rc=$?
    echo "$tool $case rc=$rc $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY|Hazard|error' $S/$tool.$case.log | tail -1)" >> $S/summary.txt
  done
done
cat $S/summary.txt
