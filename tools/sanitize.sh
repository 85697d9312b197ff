#!/bin/bash
# compute-sanitizer over a small mixed workload (single, misaligned, dense/group
# path, batch, host-streamed).  Run on a GPU box: bash tools/sanitize.sh
set -u
for tool in memcheck racecheck synccheck initcheck; do
  /usr/local/cuda/bin/compute-sanitizer --tool $tool --error-exitcode 9 python tools/sanitize_workload.py \
    > gpurun_out/san_$tool.log 2>&1
  echo "$tool rc=$?"; tail -1 gpurun_out/san_$tool.log
done
# the separate report kernel (K2) instead of K1's fused tail
for tool in racecheck synccheck; do
  ARCV_FUSED=0 /usr/local/cuda/bin/compute-sanitizer --tool $tool --error-exitcode 9 python tools/sanitize_workload.py \
    > gpurun_out/san_${tool}_k2.log 2>&1
  echo "$tool (ARCV_FUSED=0) rc=$?"; tail -1 gpurun_out/san_${tool}_k2.log
done
