#!/bin/bash
set -u
TAG=${1:-r02u}
O=gpurun_out
mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "upload or graph or pipeline" > $O/tests_up_$TAG.log 2>&1
for T in "" "--tune UPLOAD_NO_PDL=1" "" "--tune UPLOAD_NO_PDL=1"; do
  echo "tune=[$T]" >> $O/bench_up_$TAG.jsonl
  timeout 300 python bench.py --steps 10 --no-cpu-baseline --no-forward --batch 0 --no-configs $T >> $O/bench_up_$TAG.jsonl 2>> $O/bench_up_$TAG.err
done
echo done
