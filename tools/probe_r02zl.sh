#!/bin/bash
# MSV: branch-free first pass for every lane geometry (no per-word vote for Q <= 8) + the next
# batch claimed before the current one is scored.  Parity, then the default build against
# MSV_NO_PREFETCH and MSV_WORD_VOTE builds on configs 2, 3 and the config-5 M = 100 shard.
set -u
TAG=${1:-r02zl}
O=gpurun_out
mkdir -p $O
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_batch.py tests/test_gpu_fuzz.py -q -x \
  -k "msv or pipeline or fuzz or batch or config or vit" > $O/tests_msv_$TAG.log 2>&1
run() {
  local tag=$1
  for c in "--config 3" "--config 2" "--config 5 --which 0 --nseq 1250000" "--config 5 --which 1 --nseq 1250000"; do
    echo "build=$tag $c" >> $O/cmp_$TAG.jsonl
    timeout 300 python bench.py $c --steps 10 --no-cpu-baseline --no-e2e --no-forward --batch 0 --no-configs \
      >> $O/cmp_$TAG.jsonl 2>> $O/cmp_$TAG.err
  done
}
run default
HMG_NVCC_EXTRA=-DMSV_NO_PREFETCH python -c "from paper_conf_ipps_jiangg15_b200 import build; build.build(force=True)"
run noprefetch
HMG_NVCC_EXTRA=-DMSV_WORD_VOTE python -c "from paper_conf_ipps_jiangg15_b200 import build; build.build(force=True)"
run wordvote
python -c "from paper_conf_ipps_jiangg15_b200 import build; build.build(force=True)"
run default2
echo "done $TAG"
