#!/bin/bash
# Lazy-F improvement test as VIADD.16x2 + LOP3 (default) vs VIMNMX + ISETP (PAIR_IMP_VMAX): parity of
# the pair / wide kernels, configs 3 / 4 / 5 (M = 500)
set -u
TAG=${1:-r02zzj}
O=gpurun_out
mkdir -p $O
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fuzz.py -q -x -k "vit or pipeline or fuzz or config4" > $O/tests_$TAG.log 2>&1
run() {
  local tag=$1
  for c in "--config 3" "--config 5 --which 1 --nseq 1250000" "--config 4 --steps 3"; do
    echo "build=$tag $c" >> $O/cmp_$TAG.jsonl
    timeout 300 python bench.py $c --batch 0 --no-cpu-baseline --no-e2e --no-forward --no-configs \
      >> $O/cmp_$TAG.jsonl 2>> $O/cmp_$TAG.err
  done
}
run default
HMG_NVCC_EXTRA=-DPAIR_IMP_VMAX python -c "from paper_conf_ipps_jiangg15_b200 import build; build.build(force=True)"
run vmax
python -c "from paper_conf_ipps_jiangg15_b200 import build; build.build(force=True)"
run default2
echo "done $TAG"
