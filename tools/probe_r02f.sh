#!/bin/bash
set -u
TAG=${1:-r02f}
O=gpurun_out
mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "block_pair or block_kernel or calibrate" > $O/tests_cpair2_$TAG.log 2>&1
timeout 600 python tools/cpair2_bench.py 100000 2048 > $O/cpair2_$TAG.jsonl 2>&1
timeout 600 python tools/cpair2_bench.py 100000 1500 >> $O/cpair2_$TAG.jsonl 2>&1
timeout 900 python -m pytest tests/test_gpu_dist.py -q -x > $O/tests_dist_$TAG.log 2>&1
echo done
