#!/bin/bash
# e2e (hmg_pipeline_upload) vs the upload schedule: HMG_UPLOAD_GATED (1: one MSV launch whose batches
# wait on per-part landing flags; 0: one MSV launch per part), HMG_UPLOAD_PARTS parts after a 5%
# first part, sizes in geometric ratio HMG_UPLOAD_GROW/1000.  Usage (under gpurun): bash tools/upload_sweep.sh <tag> [list]
TAG=${1:-r01}
LIST=${2:-"0,6,1000 1,6,1000 1,8,1000 1,12,1000 1,12,850 1,8,1200"}
O=gpurun_out
mkdir -p $O
for GPG in $LIST; do
  IFS=, read GT P G <<< "$GPG"
  echo -n "gated=$GT,P=$P,G=$G " >> $O/upload_sweep_$TAG.jsonl
  HMG_UPLOAD_GATED=$GT HMG_UPLOAD_PARTS=$P HMG_UPLOAD_GROW=$G timeout 300 python bench.py --steps 10 --warmup 3 \
    --no-cpu-baseline --batch 0 --no-forward >> $O/upload_sweep_$TAG.jsonl 2>> $O/upload_sweep_$TAG.err
done
