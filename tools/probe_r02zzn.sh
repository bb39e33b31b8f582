#!/bin/bash
# Programmatic launch of the long-lane Viterbi after the chunked MSV (placed on the SMs the chunk
# kernel's tail frees; griddepcontrol.wait before reading its results) vs LONG_NO_PDL: parity, then
# configs 3 / 5 (M = 100, 500) and the e2e upload path
set -u
TAG=${1:-r02zzn}
O=gpurun_out
mkdir -p $O
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_dist.py -q -x -k "long_lane or pipeline or graph or upload or dist" > $O/tests_$TAG.log 2>&1
run() {
  local tag=$1
  for c in "--config 3" "--config 5 --which 0 --nseq 1250000 --no-e2e" "--config 5 --which 1 --nseq 1250000 --no-e2e"; do
    echo "build=$tag $c" >> $O/cmp_$TAG.jsonl
    timeout 300 python bench.py $c --batch 0 --steps 10 --no-cpu-baseline --no-forward --no-configs \
      >> $O/cmp_$TAG.jsonl 2>> $O/cmp_$TAG.err
  done
}
run pdl
HMG_NVCC_EXTRA=-DLONG_NO_PDL python -c "from paper_conf_ipps_jiangg15_b200 import build; build.build(force=True)"
run nopdl
python -c "from paper_conf_ipps_jiangg15_b200 import build; build.build(force=True)"
run pdl2
echo "done $TAG"
