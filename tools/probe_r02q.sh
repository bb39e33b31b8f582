#!/bin/bash
set -u
TAG=${1:-r02q}
O=gpurun_out
mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_forward.py -q -x > $O/tests_fwd_$TAG.log 2>&1
timeout 600 python tools/fwd_split_bench.py > $O/fwd_split_$TAG.jsonl 2> $O/fwd_split_$TAG.err
echo done
