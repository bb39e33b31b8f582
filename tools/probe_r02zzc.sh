#!/bin/bash
# MSV: 2GQ >= M (node M's cell through the carry into R; Q 26 -> 25 at M = 400) and the last
# 4-register chunk as int8 (LDS.64): parity, then default vs MSV_NO_BYTE4 vs MSV_Q_PLUS1 on configs
# 2 / 3 / 5 (M = 100, 500) and the f4 batch; ncu of the config-3 MSV kernel
set -u
TAG=${1:-r02zzc}
O=gpurun_out
mkdir -p $O
timeout 1800 python -m pytest tests/test_gpu_parity.py tests/test_gpu_batch.py tests/test_gpu_fuzz.py -q -x \
  -k "msv or pipeline or fuzz or batch or config" > $O/tests_$TAG.log 2>&1
run() {
  local tag=$1
  for c in "--config 3 --batch 0" "--config 2 --batch 64" "--config 5 --which 0 --nseq 1250000 --batch 0" "--config 5 --which 1 --nseq 1250000 --batch 0"; do
    echo "build=$tag $c" >> $O/cmp_$TAG.jsonl
    timeout 300 python bench.py $c --steps 10 --no-cpu-baseline --no-e2e --no-forward --no-configs \
      >> $O/cmp_$TAG.jsonl 2>> $O/cmp_$TAG.err
  done
}
run default
B="python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e --no-graph --no-configs --no-forward --batch 0"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:msv_fast -s 3 -c 1 \
  -o $O/msv_fast_$TAG -f $B > $O/ncu_full_msv_fast_$TAG.log 2>&1
python tools/ncu_summary.py $O/msv_fast_$TAG.ncu-rep > $O/ncu_full_$TAG.md 2>&1
ncu -i $O/msv_fast_$TAG.ncu-rep --page source --csv --print-source sass > $O/src_msv_fast_$TAG.csv 2>/dev/null
HMG_NVCC_EXTRA=-DMSV_NO_BYTE4 python -c "from paper_conf_ipps_jiangg15_b200 import build; build.build(force=True)"
run nobyte4
HMG_NVCC_EXTRA=-DMSV_Q_PLUS1 python -c "from paper_conf_ipps_jiangg15_b200 import build; build.build(force=True)"
run qplus1
python -c "from paper_conf_ipps_jiangg15_b200 import build; build.build(force=True)"
run default2
mkdir -p /tmp/ncu_reps_$TAG
mv $O/*_$TAG.ncu-rep /tmp/ncu_reps_$TAG/ 2>/dev/null
echo "done $TAG"
