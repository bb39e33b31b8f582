#!/bin/bash
# MSV lane-group size after 2GQ >= M (tighter fits): configs 2 (M = 200) and 5 (M = 100, 500) at
# G = 4 / 8 / 16 against the default
set -u
TAG=${1:-r02zzg}
O=gpurun_out
mkdir -p $O
for c in "--config 2" "--config 5 --which 0 --nseq 1250000" "--config 5 --which 1 --nseq 1250000"; do
  for T in "" "--tune MSV_G=4" "--tune MSV_G=8" "--tune MSV_G=16"; do
    echo "$c tune=[$T]" >> $O/geom_$TAG.jsonl
    timeout 300 python bench.py $c --batch 0 --steps 10 --no-cpu-baseline --no-e2e --no-forward --no-configs $T \
      >> $O/geom_$TAG.jsonl 2>> $O/geom_$TAG.err
  done
done
echo "done $TAG"
