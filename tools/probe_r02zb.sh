#!/bin/bash
# vit_wide with tensor-memory transitions: ncu --set full at M = 2048 (stall reasons)
set -u
TAG=${1:-r02zb}
O=gpurun_out
mkdir -p $O
M=2048
timeout 600 ncu --set full --clock-control none --import-source on -k regex:vit_wide -c 1 \
  -o $O/vit_widetm_${M}_$TAG -f python tools/vit_one.py $M 20000 VIT_WIDE=2 > $O/ncu_full_vit_widetm_${M}_$TAG.log 2>&1
python tools/ncu_summary.py $O/vit_widetm_${M}_$TAG.ncu-rep > $O/ncu_vit_widetm_${M}_$TAG.md 2>&1
ncu -i $O/vit_widetm_${M}_$TAG.ncu-rep --page raw --csv > $O/vit_widetm_raw_${M}_$TAG.csv 2>/dev/null
ncu -i $O/vit_widetm_${M}_$TAG.ncu-rep --page source --csv --print-source sass > $O/vit_widetm_src_${M}_$TAG.csv 2>/dev/null
echo "done $TAG"
