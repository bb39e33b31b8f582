#!/bin/bash
# Viterbi pair kernel: the 6-row word body unrolled (default) vs one row per loop iteration
# (VIT_ROW_NOUNROLL: no register copies at the unrolled rows' control-flow joins), configs 3 / 5
set -u
TAG=${1:-r02zzh}
O=gpurun_out
mkdir -p $O
run() {
  local tag=$1
  for c in "--config 3" "--config 5 --which 1 --nseq 1250000" "--config 5 --which 0 --nseq 1250000"; do
    echo "build=$tag $c" >> $O/cmp_$TAG.jsonl
    timeout 300 python bench.py $c --batch 0 --steps 10 --no-cpu-baseline --no-e2e --no-forward --no-configs \
      >> $O/cmp_$TAG.jsonl 2>> $O/cmp_$TAG.err
  done
}
run default
HMG_NVCC_EXTRA=-DVIT_ROW_NOUNROLL python -c "from paper_conf_ipps_jiangg15_b200 import build; build.build(force=True)"
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "vit_pair or pipeline_config3 or vit_model" > $O/tests_$TAG.log 2>&1
run nounroll
python -c "from paper_conf_ipps_jiangg15_b200 import build; build.build(force=True)"
run default2
echo "done $TAG"
