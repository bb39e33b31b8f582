#!/bin/bash
# e2e (hmg_pipeline_upload) vs the upload part schedule: HMG_UPLOAD_PARTS parts after a 5% first
# part, sizes in geometric ratio HMG_UPLOAD_GROW/1000.  Usage (under gpurun): bash tools/upload_sweep.sh <tag>
TAG=${1:-r01}
O=gpurun_out
mkdir -p $O
for PG in 6,1000 8,1000 8,850 8,700 10,850 10,750 12,900 12,800 6,750; do
  P=${PG%,*}; G=${PG#*,}
  echo -n "P=$P,G=$G " >> $O/upload_sweep_$TAG.jsonl
  HMG_UPLOAD_PARTS=$P HMG_UPLOAD_GROW=$G timeout 300 python bench.py --steps 10 --warmup 3 \
    --no-cpu-baseline --batch 0 --no-forward >> $O/upload_sweep_$TAG.jsonl 2>> $O/upload_sweep_$TAG.err
done
