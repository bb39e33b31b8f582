#!/bin/bash
# compute-sanitizer memcheck / racecheck / synccheck on a small pipeline run.
O=gpurun_out; mkdir -p $O; TAG=${1:-r01}
for tool in memcheck racecheck synccheck; do
  timeout 900 compute-sanitizer --tool $tool --error-exitcode 9 python tools/sanitize_case.py > $O/sanitize_${tool}_$TAG.log 2>&1
  echo "$tool rc=$?"; tail -3 $O/sanitize_${tool}_$TAG.log
done
