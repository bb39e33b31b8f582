#!/bin/bash
# vit_wide (one warp per sequence, shared-memory transitions): ncu --set full at M = 2048 and 1500
set -u
TAG=${1:-r02y}
O=gpurun_out
mkdir -p $O
for M in 2048 1500; do
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:vit_wide -c 1 \
    -o $O/vit_wide_${M}_$TAG -f python tools/vit_one.py $M 20000 VIT_WIDE=1 > $O/ncu_full_vit_wide_${M}_$TAG.log 2>&1
  python tools/ncu_summary.py $O/vit_wide_${M}_$TAG.ncu-rep > $O/ncu_vit_wide_${M}_$TAG.md 2>&1
  ncu -i $O/vit_wide_${M}_$TAG.ncu-rep --page source --csv --print-source sass > $O/vit_wide_src_${M}_$TAG.csv 2>/dev/null
done
echo "done $TAG"
