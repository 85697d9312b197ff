#!/bin/bash
# compute-sanitizer over a small mixed workload (single, misaligned, dense/group
# path, batch, host-streamed).  Run on a GPU box: bash tools/sanitize.sh
set -u
for tool in memcheck racecheck synccheck initcheck; do
  /usr/local/cuda/bin/compute-sanitizer --tool $tool --error-exitcode 9 python tools/sanitize_workload.py \
    > gpurun_out/san_$tool.log 2>&1
  echo "$tool rc=$?"; tail -1 gpurun_out/san_$tool.log
done
