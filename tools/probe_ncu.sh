#!/bin/bash
# One ncu --set full capture (source counters) of the first kernel matching REGEX in CMD, plus a
# metric summary and the per-instruction SASS csv.  usage: bash tools/probe_ncu.sh TAG REGEX CMD...
set -u
TAG=$1; K=$2; shift 2
O=gpurun_out
mkdir -p $O
timeout 900 ncu --set full --clock-control none --import-source on -k regex:$K -c 1 -o $O/$TAG -f "$@" > $O/ncu_$TAG.log 2>&1
python tools/ncu_summary.py $O/$TAG.ncu-rep > $O/ncu_$TAG.md 2>&1
ncu -i $O/$TAG.ncu-rep --page source --csv --print-source sass > $O/src_$TAG.csv 2>/dev/null
