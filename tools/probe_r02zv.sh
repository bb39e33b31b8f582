#!/bin/bash
# Long lane for models of <= 128 nodes: the s16x2 pair lane on G = 32 tables of its own (default) vs
# the s32 latency lane (LONG_PAIR_SMALL=0); long-lane parity; dependent-op latencies (tools/oplat.cu)
set -u
TAG=${1:-r02zv}
O=gpurun_out
mkdir -p $O
./tools/oplat > $O/oplat_$TAG.jsonl 2>&1
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fuzz.py -q -x -k "long_lane or pipeline or fuzz" > $O/tests_$TAG.log 2>&1
for T in "" "LONG_PAIR_SMALL=0"; do
  echo "tune=[$T]" >> $O/longlat_$TAG.jsonl
  timeout 600 python tools/long_latency.py 30000 $T >> $O/longlat_$TAG.jsonl 2>> $O/longlat_$TAG.err
  TT=""; [ -n "$T" ] && TT="--tune $T"
  for c in "--config 5 --which 0 --nseq 1250000" "--config 1"; do
    echo "tune=[$T] $c" >> $O/cmp_$TAG.jsonl
    timeout 300 python bench.py $c --batch 0 --steps 10 --no-cpu-baseline --no-e2e --no-forward --no-configs $TT \
      >> $O/cmp_$TAG.jsonl 2>> $O/cmp_$TAG.err
  done
done
echo "done $TAG"
