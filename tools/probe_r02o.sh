#!/bin/bash
set -u
TAG=${1:-r02o}
O=gpurun_out
mkdir -p $O
for T in "" "--tune VIT_PAIR_G=16" "--tune PIPE_LONG_SMS=4" "--tune PIPE_LONG_SMS=8" "--tune MSV_G=16" "--tune MSV_G=4" "--tune VIT_SCAN=1" ""; do
  echo "tune=[$T]" >> $O/bench_sweep_$TAG.jsonl
  timeout 300 python bench.py --steps 10 --no-cpu-baseline --no-e2e --no-forward --batch 0 --no-configs $T >> $O/bench_sweep_$TAG.jsonl 2>> $O/bench_sweep_$TAG.err
done
timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none -k regex:vit_cpair2 -c 1 \
  --csv --log-file $O/ncu_c4_traffic_$TAG.csv python tools/vit_one.py 2048 550000 > $O/ncu_c4_traffic_$TAG.log 2>&1
echo done
