#!/bin/bash
set -u
TAG=${1:-r02g}
O=gpurun_out
mkdir -p $O
timeout 300 python __graft_entry__.py smoke > $O/smoke_$TAG.log 2>&1
timeout 1500 python -m pytest tests -q -m gpu -x > $O/gpu_tests_$TAG.log 2>&1
timeout 600 python tools/cpair2_bench.py 100000 2048 > $O/cpair2_$TAG.jsonl 2>&1
timeout 900 python bench.py > $O/bench_$TAG.json 2> $O/bench_$TAG.err
timeout 600 python bench.py --config 4 --steps 3 --no-cpu-baseline > $O/bench_c4_$TAG.json 2> $O/bench_c4_$TAG.err
echo done
