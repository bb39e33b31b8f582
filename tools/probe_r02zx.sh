#!/bin/bash
# e2e upload schedule after the MSV speed-up (MSV now consumes ~40 M residues/ms against ~80 M/ms of
# H2D): parts / first part (permille) / geometric growth of hmg_pipeline_upload, config 3 e2e.
# usage: PARTS="6,50,1000 4,50,1000,2" bash tools/probe_r02zx.sh <tag>
set -u
TAG=${1:-r02zx}
PARTS=${PARTS:-"6,50,1000 8,20,1500 8,20,2000 10,20,1500 12,10,1500 6,20,1500 8,50,1500 4,50,1000 6,50,1000"}
O=gpurun_out
mkdir -p $O
[ -n "${TESTS:-}" ] && timeout 1500 python -m pytest tests/test_gpu_parity.py -q -x -k "upload or graph" > $O/tests_$TAG.log 2>&1
for P in $PARTS; do
  IFS=, read -r NP FP GR NS <<< "$P"
  NS=${NS:-1}
  echo "parts=$NP first=$FP grow=$GR streams=$NS" >> $O/e2e_$TAG.jsonl
  timeout 300 python bench.py --batch 0 --steps 10 --no-cpu-baseline --no-forward --no-configs \
    --tune UPLOAD_PARTS=$NP --tune UPLOAD_FIRST_PERMILLE=$FP --tune UPLOAD_GROW=$GR --tune UPLOAD_MSV_STREAMS=$NS >> $O/e2e_$TAG.jsonl 2>> $O/e2e_$TAG.err
done
echo "done $TAG"
