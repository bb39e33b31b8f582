#!/bin/bash
# Config-3 Viterbi stage on the long-model kernels: two warps per sequence without a row barrier
# (vit_cpair2, Q = 4) and one warp per sequence with shared-memory transitions (vit_wide, Q = 8),
# against the lane-group pair kernel; the Forward stage with two warps per sequence (FWD_W = 2)
set -u
TAG=${1:-r02zze}
O=gpurun_out
mkdir -p $O
for T in "" "--tune VIT_PAIR_CTA=1 --tune VIT_WIDE=0" "--tune VIT_PAIR_CTA=1" "--tune VIT_PAIR_CTA=1 --tune VIT_WIDE=0 --tune VIT_CPAIR2=0" ""; do
  echo "tune=[$T]" >> $O/cmp_$TAG.jsonl
  timeout 300 python bench.py --batch 0 --steps 10 --no-cpu-baseline --no-e2e --no-forward --no-configs $T \
    >> $O/cmp_$TAG.jsonl 2>> $O/cmp_$TAG.err
done
for T in "" "--tune FWD_W=2" "--tune FWD_W=2 --tune FWD_QMAX=8"; do
  echo "fwd tune=[$T]" >> $O/fwd_$TAG.jsonl
  timeout 300 python bench.py --batch 0 --steps 5 --no-cpu-baseline --no-e2e --no-configs $T \
    >> $O/fwd_$TAG.jsonl 2>> $O/fwd_$TAG.err
done
echo "done $TAG"
