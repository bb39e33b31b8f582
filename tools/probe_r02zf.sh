#!/bin/bash
set -u
TAG=${1:-r02zf}
O=gpurun_out
mkdir -p $O
timeout 1500 python -m pytest tests -m gpu -q > $O/gpu_tests_$TAG.log 2>&1
timeout 300 python __graft_entry__.py smoke > $O/smoke_$TAG.log 2>&1
timeout 600 python tools/wide_mid_bench.py 100000 600 800 1000 > $O/wide_mid_$TAG.jsonl 2>&1
echo "done $TAG"
