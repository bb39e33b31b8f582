#!/bin/bash
# vit_wide (TMEM) as the config-4 default: full GPU suite, config-4 bench, ncu DRAM traffic of the
# config-4 launch and one ncu --set full capture (source counters for the SASS mix)
set -u
TAG=${1:-r02ze}
O=gpurun_out
mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,clocks_event_reasons.active --format=csv > $O/nvsmi_$TAG.txt 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q > $O/gpu_tests_$TAG.log 2>&1
timeout 900 python bench.py --config 4 --steps 3 > $O/bench_c4_$TAG.json 2> $O/bench_c4_$TAG.err
timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none -k regex:vit_wide -c 1 \
  --csv --log-file $O/ncu_c4_traffic_$TAG.csv python tools/vit_one.py 2048 550000 > $O/ncu_c4_traffic_$TAG.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:vit_wide -c 1 \
  -o $O/vit_wide_$TAG -f python tools/vit_one.py 2048 100000 > $O/ncu_full_vit_wide_$TAG.log 2>&1
python tools/ncu_summary.py $O/vit_wide_$TAG.ncu-rep > $O/ncu_vit_wide_$TAG.md 2>&1
ncu -i $O/vit_wide_$TAG.ncu-rep --page source --csv --print-source sass > $O/src_vit_wide_$TAG.csv 2>/dev/null
mkdir -p /tmp/ncu_reps_$TAG; mv $O/vit_wide_$TAG.ncu-rep /tmp/ncu_reps_$TAG/
echo "done $TAG"
