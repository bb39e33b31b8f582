#!/bin/bash
# MSV: conflict-free remainder chunks (per-group copies) + rows stopped at the group's last word:
# MSV parity (parity, batch, fuzz), stage timing on configs 3 and 2, ncu of the config-3 MSV kernel
set -u
TAG=${1:-r02zk}
O=gpurun_out
mkdir -p $O
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_batch.py tests/test_gpu_fuzz.py -q -x \
  -k "msv or pipeline or fuzz or batch or config or vit" > $O/tests_msv_$TAG.log 2>&1
timeout 600 python tools/stage_bench.py 3 5 > $O/stage3_$TAG.jsonl 2>&1
timeout 600 python tools/stage_bench.py 2 3 > $O/stage2_$TAG.jsonl 2>&1
B="python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e --no-graph --no-configs --no-forward --batch 0"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:msv_fast -s 3 -c 1 \
  -o $O/msv_fast_$TAG -f $B > $O/ncu_full_msv_fast_$TAG.log 2>&1
python tools/ncu_summary.py $O/msv_fast_$TAG.ncu-rep > $O/ncu_full_$TAG.md 2>&1
ncu -i $O/msv_fast_$TAG.ncu-rep --page source --csv --print-source sass > $O/src_msv_fast_$TAG.csv 2>/dev/null
mkdir -p /tmp/ncu_reps_$TAG
mv $O/*_$TAG.ncu-rep /tmp/ncu_reps_$TAG/ 2>/dev/null
echo "done $TAG"
