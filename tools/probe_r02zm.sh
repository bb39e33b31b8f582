#!/bin/bash
# MSV short rows: per-word vote only for whole-warp batches (default) vs for every Q <= 8 geometry
# (MSV_WORD_VOTE_ALL): parity, then configs 2, 3, 5 (M = 100 / 500 shards) and the f4 batch leg.
set -u
TAG=${1:-r02zm}
O=gpurun_out
mkdir -p $O
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_batch.py tests/test_gpu_fuzz.py -q -x \
  -k "msv or pipeline or fuzz or batch or config or vit" > $O/tests_msv_$TAG.log 2>&1
run() {
  local tag=$1
  for c in "--config 2 --batch 64" "--config 3 --batch 0" "--config 5 --which 0 --nseq 1250000 --batch 0" "--config 5 --which 1 --nseq 1250000 --batch 0"; do
    echo "build=$tag $c" >> $O/cmp_$TAG.jsonl
    timeout 300 python bench.py $c --steps 10 --no-cpu-baseline --no-e2e --no-forward --no-configs \
      >> $O/cmp_$TAG.jsonl 2>> $O/cmp_$TAG.err
  done
}
run default
HMG_NVCC_EXTRA=-DMSV_WORD_VOTE_ALL python -c "from paper_conf_ipps_jiangg15_b200 import build; build.build(force=True)"
run wordvote_all
python -c "from paper_conf_ipps_jiangg15_b200 import build; build.build(force=True)"
run default2
echo "done $TAG"
