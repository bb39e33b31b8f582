#!/bin/bash
set -u
TAG=${1:-r02k}
O=gpurun_out
mkdir -p $O
timeout 300 python __graft_entry__.py smoke > $O/smoke_$TAG.log 2>&1
timeout 2400 python -m pytest tests -q -m gpu > $O/gpu_tests_$TAG.log 2>&1
bash tools/sanitize.sh $TAG > /dev/null 2>&1
echo done
