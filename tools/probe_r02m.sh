#!/bin/bash
set -u
TAG=${1:-r02m}
O=gpurun_out
mkdir -p $O
timeout 300 python __graft_entry__.py smoke > $O/smoke_$TAG.log 2>&1
timeout 2400 python -m pytest tests -q -m gpu > $O/gpu_tests_$TAG.log 2>&1
for T in "--tune NO_SURV_QUEUE=1" "" "--tune PIPE_LONG_SMS=8" "--tune PIPE_LONG_SMS=24" "--tune PIPE_LONG_SMS=32" "--tune NO_SURV_QUEUE=1"; do
  echo "tune=[$T]" >> $O/bench_vq_$TAG.jsonl
  timeout 300 python bench.py --steps 10 --no-cpu-baseline --no-e2e --no-forward --batch 0 --no-configs $T >> $O/bench_vq_$TAG.jsonl 2>> $O/bench_vq_$TAG.err
done
timeout 600 python tools/cpair2_bench.py 100000 2048 > $O/cpair2_$TAG.jsonl 2>&1
echo done
