#!/bin/bash
# MSV rows without the per-row update branch (checked re-run on hits): parity + stage timing + bench
set -u
TAG=${1:-r02zi}
O=gpurun_out
mkdir -p $O
timeout 1500 python -m pytest tests -m gpu -q -x > $O/gpu_tests_$TAG.log 2>&1
timeout 600 python tools/stage_bench.py 3 5 > $O/stage_$TAG.jsonl 2>&1
timeout 900 python bench.py --no-cpu-baseline > $O/bench_$TAG.json 2> $O/bench_$TAG.err
echo "done $TAG"
