#!/bin/bash
# Long lane: per-QL fallback variant (word vote for QL <= 4, checked pass above) on configs 2/3/5,
# and the long-lane Viterbi with the max-plus scan Lazy-F (LONG_SCAN) vs vote-terminated passes
set -u
TAG=${1:-r02zu}
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
run default
HMG_NVCC_EXTRA=-DLONG_SCAN python -c "from paper_conf_ipps_jiangg15_b200 import build; build.build(force=True)"
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "long_lane or pipeline_config" > $O/tests_scan_$TAG.log 2>&1
run scan
python -c "from paper_conf_ipps_jiangg15_b200 import build; build.build(force=True)"
echo "done $TAG"
