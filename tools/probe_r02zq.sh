#!/bin/bash
# Long-lane Viterbi row latency: row_lat (default) vs row (LONG_ROW_PLAIN) on one 30k-residue sequence
set -u
TAG=${1:-r02zq}
O=gpurun_out
mkdir -p $O
echo "build=lat" >> $O/longlat_$TAG.jsonl
timeout 600 python tools/long_latency.py 30000 >> $O/longlat_$TAG.jsonl 2>> $O/longlat_$TAG.err
HMG_NVCC_EXTRA=-DLONG_ROW_PLAIN python -c "from paper_conf_ipps_jiangg15_b200 import build; build.build(force=True)"
echo "build=plain" >> $O/longlat_$TAG.jsonl
timeout 600 python tools/long_latency.py 30000 >> $O/longlat_$TAG.jsonl 2>> $O/longlat_$TAG.err
for c in "--config 5 --which 0 --nseq 1250000" "--config 3"; do
  echo "build=plain $c" >> $O/cmp_$TAG.jsonl
  timeout 300 python bench.py $c --batch 0 --steps 10 --no-cpu-baseline --no-e2e --no-forward --no-configs \
    >> $O/cmp_$TAG.jsonl 2>> $O/cmp_$TAG.err
done
python -c "from paper_conf_ipps_jiangg15_b200 import build; build.build(force=True)"
echo "done $TAG"
