#!/bin/bash
# Probe: config-4 Viterbi (vit_cpair) timing + one ncu --set full capture with source counters.
# usage (under gpurun): bash tools/probe_cpair.sh <tag> [nseq]
set -u
TAG=${1:-r02a}
N=${2:-20000}
O=gpurun_out
mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,clocks_event_reasons.active --format=csv > $O/nvsmi_$TAG.txt 2>&1
timeout 300 python __graft_entry__.py smoke > $O/smoke_$TAG.log 2>&1
timeout 300 python tools/vit_one.py 2048 550000 > $O/vit_one_$TAG.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:vit_c -c 1 \
  -o $O/vit_cpair_$TAG -f python tools/vit_one.py 2048 $N > $O/ncu_full_vit_cpair_$TAG.log 2>&1
python tools/ncu_summary.py $O/vit_cpair_$TAG.ncu-rep > $O/ncu_vit_cpair_$TAG.md 2>&1
ncu -i $O/vit_cpair_$TAG.ncu-rep --page source --csv --print-source sass > $O/vit_cpair_src_$TAG.csv 2>/dev/null
echo "done $TAG"
