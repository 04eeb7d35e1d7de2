#!/bin/bash
# round-2 GPU check: build, the -m gpu suite with durations, one short bench line
cd "$GRAFT_REPO_ROOT"
make -j32 -s 2>&1 | tail -3
timeout 1500 python -m pytest tests -m gpu -x -q --durations=15 "$@" > gpurun_out/r2_gpu_tests.log 2>&1
echo "pytest rc=$?" >> gpurun_out/r2_gpu_tests.log
tail -30 gpurun_out/r2_gpu_tests.log
