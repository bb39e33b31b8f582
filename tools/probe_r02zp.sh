#!/bin/bash
# Long-lane Viterbi in the latency row form (VitPairLane::row_lat: diagonal carries exchanged with the
# first Lazy-F carry, one REDUX.OR for the hit and Lazy-F votes, emissions a row ahead): parity, then
# configs 3 / 5 (M = 100, 500 shards); VIT_PAIR_LAT builds also run the main G = 32 pair kernel that way.
set -u
TAG=${1:-r02zp}
O=gpurun_out
mkdir -p $O
timeout 1800 python -m pytest tests/test_gpu_parity.py tests/test_gpu_batch.py tests/test_gpu_fuzz.py tests/test_gpu_dist.py -q -x \
  -k "pipeline or fuzz or batch or config or vit or dist" > $O/tests_$TAG.log 2>&1
run() {
  local tag=$1
  for c in "--config 5 --which 0 --nseq 1250000" "--config 3" "--config 5 --which 1 --nseq 1250000"; do
    echo "build=$tag $c" >> $O/cmp_$TAG.jsonl
    timeout 300 python bench.py $c --batch 0 --steps 10 --no-cpu-baseline --no-e2e --no-forward --no-configs \
      >> $O/cmp_$TAG.jsonl 2>> $O/cmp_$TAG.err
  done
}
run default
HMG_NVCC_EXTRA=-DVIT_PAIR_LAT python -c "from paper_conf_ipps_jiangg15_b200 import build; build.build(force=True)"
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "vit_pair or pipeline_config3 or vit_model" > $O/tests_lat_$TAG.log 2>&1
run vitlat
python -c "from paper_conf_ipps_jiangg15_b200 import build; build.build(force=True)"
run default2
echo "done $TAG"
