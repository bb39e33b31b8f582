#!/bin/bash
# Long-lane sequential MSV fallback: checked pass only (default) vs per-word vote (LONG_FALLBACK_WV)
# vs branch-free + checked re-run (LONG_FALLBACK_BF) on configs 2, 3, 5 (M = 100 / 500 shards);
# the long-lane latency split (MSV alone vs pipeline) on one 30k-residue sequence
set -u
TAG=${1:-r02zt}
O=gpurun_out
mkdir -p $O
timeout 1500 python -m pytest tests/test_gpu_parity.py -q -x -k "long_lane or msv or config" > $O/tests_$TAG.log 2>&1
run() {
  local tag=$1
  echo "build=$tag" >> $O/longlat_$TAG.jsonl
  timeout 600 python tools/long_latency.py 30000 >> $O/longlat_$TAG.jsonl 2>> $O/longlat_$TAG.err
  for c in "--config 2" "--config 3" "--config 5 --which 0 --nseq 1250000" "--config 5 --which 1 --nseq 1250000"; do
    echo "build=$tag $c" >> $O/cmp_$TAG.jsonl
    timeout 300 python bench.py $c --batch 0 --steps 10 --no-cpu-baseline --no-e2e --no-forward --no-configs \
      >> $O/cmp_$TAG.jsonl 2>> $O/cmp_$TAG.err
  done
}
run checked
HMG_NVCC_EXTRA=-DLONG_FALLBACK_WV python -c "from paper_conf_ipps_jiangg15_b200 import build; build.build(force=True)"
run wv
HMG_NVCC_EXTRA=-DLONG_FALLBACK_BF python -c "from paper_conf_ipps_jiangg15_b200 import build; build.build(force=True)"
run bf
python -c "from paper_conf_ipps_jiangg15_b200 import build; build.build(force=True)"
echo "done $TAG"
