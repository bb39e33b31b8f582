#!/bin/bash
# Round-2 evidence under gpurun: ncu launch list of the bench step, ncu --set full (source counters)
# of the hot kernels of every BASELINE config leg (config-3 MSV + Viterbi stage + long lane, config-4
# two-warp Viterbi, f4 batch MSV), their summaries and executed SASS mixes per cell.
# usage: bash tools/evidence_r02.sh <tag>
set -u
TAG=${1:-r02}
O=gpurun_out
mkdir -p $O
B="python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e --no-graph --no-configs --no-forward"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_$TAG.csv \
  python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-e2e --no-graph --batch 0 --no-forward --no-configs \
  > $O/ncu_launch_bench_$TAG.log 2>&1
python tools/launch_summary.py $O/launches_$TAG.csv "bench config 3 step ($TAG)" > $O/launches_$TAG.md 2>&1
for K in msv_fast vit_pair pipe_long_vpair; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:$K -s 3 -c 1 \
    -o $O/${K}_$TAG -f $B --batch 0 > $O/ncu_full_${K}_$TAG.log 2>&1
done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:msv_multi -c 1 \
  -o $O/msv_multi_$TAG -f $B --batch 64 > $O/ncu_full_msv_multi_$TAG.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:vit_cpair2 -c 1 \
  -o $O/vit_cpair2_$TAG -f python tools/vit_one.py 2048 100000 > $O/ncu_full_vit_cpair2_$TAG.log 2>&1
python tools/ncu_summary.py $O/*_$TAG.ncu-rep > $O/ncu_full_$TAG.md 2>&1
for K in msv_fast vit_pair pipe_long_vpair msv_multi vit_cpair2; do
  ncu -i $O/${K}_$TAG.ncu-rep --page source --csv --print-source sass > $O/src_${K}_$TAG.csv 2>/dev/null
done
mkdir -p /tmp/ncu_reps_$TAG
for f in $O/*_$TAG.ncu-rep; do mv "$f" /tmp/ncu_reps_$TAG/; done
echo "done $TAG"
