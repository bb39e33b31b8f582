#!/bin/bash
# e2e (hmg_pipeline_upload) vs the upload schedule: UPLOAD_PARTS parts after a 5% first part, sizes
# in geometric ratio UPLOAD_GROW/1000 (bench.py --tune).  Usage (under gpurun): bash tools/upload_sweep.sh <tag> [list]
TAG=${1:-r02}
LIST=${2:-"6,1000 8,1000 12,1000 12,850 8,1200"}
O=gpurun_out
mkdir -p $O
for PG in $LIST; do
  IFS=, read P G <<< "$PG"
  echo -n "P=$P,G=$G " >> $O/upload_sweep_$TAG.jsonl
  timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --batch 0 --no-forward --no-configs \
    --tune UPLOAD_PARTS=$P --tune UPLOAD_GROW=$G >> $O/upload_sweep_$TAG.jsonl 2>> $O/upload_sweep_$TAG.err
done
