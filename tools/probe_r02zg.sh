#!/bin/bash
# round-2 final bench lines: default (config 3 + configs leg), reference arm, config 4, config 5
set -u
TAG=${1:-r02zg}
O=gpurun_out
mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,clocks_event_reasons.active --format=csv > $O/nvsmi_$TAG.txt 2>&1
S=$(date +%s.%N); timeout 900 python bench.py > $O/bench_$TAG.json 2> $O/bench_$TAG.err; E=$(date +%s.%N)
echo "bench wall $(echo "$E - $S" | bc)" >> $O/walls_$TAG.txt
S=$(date +%s.%N); timeout 900 python bench.py --impl reference > $O/bench_ref_$TAG.json 2> $O/bench_ref_$TAG.err; E=$(date +%s.%N)
echo "ref wall $(echo "$E - $S" | bc)" >> $O/walls_$TAG.txt
S=$(date +%s.%N); timeout 900 python bench.py --config 4 --steps 3 > $O/bench_c4_$TAG.json 2> $O/bench_c4_$TAG.err; E=$(date +%s.%N)
echo "c4 wall $(echo "$E - $S" | bc)" >> $O/walls_$TAG.txt
S=$(date +%s.%N); timeout 900 python bench.py --config 5 --which 2 --steps 3 --no-cpu-baseline > $O/bench_c5_$TAG.json 2> $O/bench_c5_$TAG.err; E=$(date +%s.%N)
echo "c5 wall $(echo "$E - $S" | bc)" >> $O/walls_$TAG.txt
echo "done $TAG"
