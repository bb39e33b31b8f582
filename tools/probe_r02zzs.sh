#!/bin/bash
# Lazy-F: in-lane steps checked before the full chain on an improving pass (K0, default 3)
set -u
TAG=${1:-r02zzs}
O=gpurun_out
mkdir -p $O
for K in 3 2 5 7 3; do
  HMG_NVCC_EXTRA=-DPAIR_K0=$K python -c "from paper_conf_ipps_jiangg15_b200 import build; build.build(force=True)"
  for c in "--config 3" "--config 5 --which 1 --nseq 1250000"; do
    echo "K0=$K $c" >> $O/k0_$TAG.jsonl
    timeout 300 python bench.py $c --batch 0 --steps 10 --no-cpu-baseline --no-e2e --no-forward --no-configs \
      >> $O/k0_$TAG.jsonl 2>> $O/k0_$TAG.err
  done
done
python -c "from paper_conf_ipps_jiangg15_b200 import build; build.build(force=True)"
echo "done $TAG"
