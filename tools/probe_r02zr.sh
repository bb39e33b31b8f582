#!/bin/bash
# Why a lone long-lane Viterbi row takes ~390 cycles (M = 400): ncu --set full with source counters of
# pipe_long_vpair_kernel on one 30k-residue sequence (tools/long_latency.py), row() and row_lat builds
set -u
TAG=${1:-r02zr}
O=gpurun_out
mkdir -p $O
for b in plain lat; do
  if [ $b = lat ]; then HMG_NVCC_EXTRA=-DLONG_ROW_LAT python -c "from paper_conf_ipps_jiangg15_b200 import build; build.build(force=True)"; fi
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:pipe_long_vpair -s 1 -c 1 \
    -o $O/longv_${b}_$TAG -f python tools/long_latency.py 30000 > $O/ncu_longv_${b}_$TAG.log 2>&1
  python tools/ncu_summary.py $O/longv_${b}_$TAG.ncu-rep > $O/ncu_longv_${b}_$TAG.md 2>&1
  ncu -i $O/longv_${b}_$TAG.ncu-rep --page source --csv --print-source sass > $O/src_longv_${b}_$TAG.csv 2>/dev/null
done
python -c "from paper_conf_ipps_jiangg15_b200 import build; build.build(force=True)"
mkdir -p /tmp/ncu_reps_$TAG
mv $O/*_$TAG.ncu-rep /tmp/ncu_reps_$TAG/ 2>/dev/null
echo "done $TAG"
