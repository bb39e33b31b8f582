#!/bin/bash
# Lane-group geometry sweeps on the other BASELINE configs (config 2 M = 200, config-5 shard
# M = 100 / 500 / 1000): MSV_G and VIT_PAIR_G against the defaults.
set -u
TAG=${1:-r02s}
O=gpurun_out
mkdir -p $O
for T in "" "--tune MSV_G=4" "--tune MSV_G=16"; do
  echo "c2 tune=[$T]" >> $O/geom_$TAG.jsonl
  timeout 300 python bench.py --config 2 --steps 5 --no-cpu-baseline $T >> $O/geom_$TAG.jsonl 2>> $O/geom_$TAG.err
done
for W in 0 1 2; do
  for T in "" "--tune MSV_G=4" "--tune MSV_G=16" "--tune VIT_PAIR_G=16" "--tune VIT_PAIR_G=8"; do
    echo "c5/$W tune=[$T]" >> $O/geom_$TAG.jsonl
    timeout 300 python bench.py --config 5 --which $W --nseq 1250000 --steps 5 --no-cpu-baseline $T >> $O/geom_$TAG.jsonl 2>> $O/geom_$TAG.err
  done
done
echo done
