#!/bin/bash
# Chunk length of the long lane's chunked MSV (PIPE_CHUNK, rows; default 1032) on configs 3 / 2 / 5
set -u
TAG=${1:-r02zzm}
O=gpurun_out
mkdir -p $O
timeout 900 python tools/sanitize_case.py > $O/allkernels_$TAG.log 2>&1
for c in "--config 3" "--config 2" "--config 5 --which 1 --nseq 1250000"; do
  for T in 1032 1500 2004 3000 1032; do
    echo "$c chunk=$T" >> $O/chunk_$TAG.jsonl
    timeout 300 python bench.py $c --batch 0 --steps 10 --no-cpu-baseline --no-e2e --no-forward --no-configs \
      --tune PIPE_CHUNK=$T >> $O/chunk_$TAG.jsonl 2>> $O/chunk_$TAG.err
  done
done
echo "done $TAG"
