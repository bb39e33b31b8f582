#!/bin/bash
# Evidence after 2GQ >= M (node M's cell through the carry into R): full GPU suite, smoke, bench lines
# (default with configs leg, reference arm, config 4, config 5 full DB), ncu of the config-3 MSV kernel
# and its SASS source counters, the bench-step launch list
set -u
TAG=${1:-r02zzq}
O=gpurun_out
mkdir -p $O
timeout 2400 python -m pytest tests -m gpu -q -x > $O/gpu_tests_$TAG.log 2>&1
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke_$TAG.log 2>&1
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,clocks_event_reasons.active --format=csv > $O/nvsmi_$TAG.txt 2>&1
timeout 900 python bench.py > $O/bench_$TAG.json 2> $O/bench_$TAG.err
timeout 900 python bench.py --impl reference > $O/bench_ref_$TAG.json 2> $O/bench_ref_$TAG.err
timeout 900 python bench.py --config 4 --steps 3 > $O/bench_c4_$TAG.json 2> $O/bench_c4_$TAG.err
timeout 900 python bench.py --config 5 --which 2 --steps 3 --no-cpu-baseline > $O/bench_c5_$TAG.json 2> $O/bench_c5_$TAG.err
B="python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e --no-graph --no-configs --no-forward --batch 0"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:msv_fast -s 3 -c 1 \
  -o $O/msv_fast_$TAG -f $B > $O/ncu_full_msv_fast_$TAG.log 2>&1
python tools/ncu_summary.py $O/msv_fast_$TAG.ncu-rep > $O/ncu_full_$TAG.md 2>&1
ncu -i $O/msv_fast_$TAG.ncu-rep --page source --csv --print-source sass > $O/src_msv_fast_$TAG.csv 2>/dev/null
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_$TAG.csv \
  python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-e2e --no-graph --batch 0 --no-forward --no-configs \
  > $O/ncu_launch_bench_$TAG.log 2>&1
python tools/launch_summary.py $O/launches_$TAG.csv "bench config 3 step ($TAG)" > $O/launches_$TAG.md 2>&1
mkdir -p /tmp/ncu_reps_$TAG
mv $O/*_$TAG.ncu-rep /tmp/ncu_reps_$TAG/ 2>/dev/null
echo "done $TAG"
