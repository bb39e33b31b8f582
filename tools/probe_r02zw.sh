#!/bin/bash
# Long-lane latency row v2 (LONG_ROW_LAT: diagonal carries shuffled with the first Lazy-F carry,
# ballot + vote issued together, no REDUX) vs row(): lone-row latency, configs 3 / 5, long-lane parity;
# the pipeline long-lane cut (PIPE_LLONG) below the default on config 3
set -u
TAG=${1:-r02zw}
O=gpurun_out
mkdir -p $O
run() {
  local tag=$1
  echo "build=$tag" >> $O/longlat_$TAG.jsonl
  timeout 600 python tools/long_latency.py 30000 >> $O/longlat_$TAG.jsonl 2>> $O/longlat_$TAG.err
  for c in "--config 3" "--config 5 --which 0 --nseq 1250000" "--config 5 --which 1 --nseq 1250000"; do
    echo "build=$tag $c" >> $O/cmp_$TAG.jsonl
    timeout 300 python bench.py $c --batch 0 --steps 10 --no-cpu-baseline --no-e2e --no-forward --no-configs \
      >> $O/cmp_$TAG.jsonl 2>> $O/cmp_$TAG.err
  done
}
run plain
for T in 1500 2000 2400; do
  echo "build=plain llong=$T" >> $O/cmp_$TAG.jsonl
  timeout 300 python bench.py --config 3 --batch 0 --steps 10 --no-cpu-baseline --no-e2e --no-forward --no-configs \
    --tune PIPE_LLONG=$T >> $O/cmp_$TAG.jsonl 2>> $O/cmp_$TAG.err
done
HMG_NVCC_EXTRA=-DLONG_ROW_LAT python -c "from paper_conf_ipps_jiangg15_b200 import build; build.build(force=True)"
timeout 1500 python -m pytest tests/test_gpu_parity.py -q -x -k "long_lane or pipeline_config" > $O/tests_lat_$TAG.log 2>&1
run lat
python -c "from paper_conf_ipps_jiangg15_b200 import build; build.build(force=True)"
echo "done $TAG"
