#!/bin/bash
set -u
TAG=${1:-r02t}
O=gpurun_out
mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "block_pair or block_kernel" > $O/tests_c2_$TAG.log 2>&1
timeout 600 python tools/cpair2_bench.py 100000 2048 > $O/cpair2_$TAG.jsonl 2>&1
bash tools/probe_r02s.sh $TAG
echo done
