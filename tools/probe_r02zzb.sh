#!/bin/bash
# Split pipeline (PIPE_SPLIT_PERMILLE): parity vs the unsplit call, then config 3 / 5 timings per split
set -u
TAG=${1:-r02zzb}
O=gpurun_out
mkdir -p $O
timeout 1500 python -m pytest tests/test_gpu_parity.py -q -x -k "split or graph or pipeline_config3" > $O/tests_$TAG.log 2>&1
for T in 0 600 700 800 900 0; do
  for c in "--config 3" "--config 5 --which 0 --nseq 1250000" "--config 5 --which 1 --nseq 1250000"; do
    echo "split=$T $c" >> $O/cmp_$TAG.jsonl
    timeout 300 python bench.py $c --batch 0 --steps 10 --no-cpu-baseline --no-e2e --no-forward --no-configs \
      --tune PIPE_SPLIT_PERMILLE=$T >> $O/cmp_$TAG.jsonl 2>> $O/cmp_$TAG.err
  done
done
echo "done $TAG"
