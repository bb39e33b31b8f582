#!/bin/bash
# Viterbi pair lane group for M <= 128 (default 16 above M = 64): G = 8 vs 16 on config 5 (M = 100)
set -u
TAG=${1:-r02zzr}
O=gpurun_out
mkdir -p $O
for T in "" "--tune VIT_PAIR_G=8" "" "--tune VIT_PAIR_G=8"; do
  echo "c5/0 tune=[$T]" >> $O/vg_$TAG.jsonl
  timeout 300 python bench.py --config 5 --which 0 --nseq 1250000 --batch 0 --steps 10 --no-cpu-baseline --no-e2e \
    --no-forward --no-configs $T >> $O/vg_$TAG.jsonl 2>> $O/vg_$TAG.err
done
echo "done $TAG"
