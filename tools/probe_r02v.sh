#!/bin/bash
set -u
TAG=${1:-r02v}
O=gpurun_out
mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "block_pair" > $O/tests_wide_$TAG.log 2>&1
for M in 2048 1500 1100; do
  timeout 600 python tools/cpair2_bench.py 100000 $M >> $O/cpair2_$TAG.jsonl 2>&1
done
echo done
