#!/bin/bash
# pipeline long-lane cut (tuning PIPE_LLONG, default max(1500, 8 x mean) = 2880 on config 3) and its
# SM count (PIPE_LONG_SMS).  Usage (under gpurun): bash tools/llong_sweep.sh <tag>
TAG=${1:-r02}
O=gpurun_out
mkdir -p $O
for CS in 2880,0 2000,0 2400,0 3500,0 5000,0 2880,12 2880,6; do
  C=${CS%,*}; S=${CS#*,}
  echo -n "llong=$C,sms=$S " >> $O/llong_sweep_$TAG.jsonl
  T="--tune PIPE_LLONG=$C"
  if [ "$S" != "0" ]; then T="$T --tune PIPE_LONG_SMS=$S"; fi
  timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e --batch 0 --no-forward --no-configs \
    $T >> $O/llong_sweep_$TAG.jsonl 2>> $O/llong_sweep_$TAG.err
done
