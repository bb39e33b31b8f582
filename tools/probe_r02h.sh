#!/bin/bash
set -u
TAG=${1:-r02h}
O=gpurun_out
mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fuzz.py tests/test_gpu_batch.py -q -x -k "msv or pipeline or fuzz or batch" > $O/tests_msvb_$TAG.log 2>&1
for T in "" "--tune MSV_NO_BYTES=1" "" "--tune MSV_NO_BYTES=1"; do
  echo "tune=[$T]" >> $O/bench_msvb_$TAG.jsonl
  timeout 300 python bench.py --steps 10 --no-cpu-baseline --no-e2e --no-forward --batch 0 --no-configs $T >> $O/bench_msvb_$TAG.jsonl 2>> $O/bench_msvb_$TAG.err
done
for T in "" "--tune MSV_NO_BYTES=1"; do
  echo "tune=[$T]" >> $O/bench_msvb_$TAG.jsonl
  timeout 300 python bench.py --config 2 --steps 10 --no-cpu-baseline $T >> $O/bench_msvb_$TAG.jsonl 2>> $O/bench_msvb_$TAG.err
done
echo done
