#!/bin/bash
# MSV upper bound: the G = 8 / Q = 26 row loop without the per-row update branch (timing only,
# -DMSV_NOCHECK_EXPERIMENT: wrong on hits) vs the normal build
set -u
TAG=${1:-r02zh}
O=gpurun_out
mkdir -p $O
timeout 600 python tools/stage_bench.py 3 5 > $O/stage_default_$TAG.jsonl 2>&1
HMG_NVCC_EXTRA=-DMSV_NOCHECK_EXPERIMENT python -c "from paper_conf_ipps_jiangg15_b200 import build; build.build(force=True)"
timeout 600 python tools/stage_bench.py 3 5 > $O/stage_nocheck_$TAG.jsonl 2>&1
python -c "from paper_conf_ipps_jiangg15_b200 import build; build.build(force=True)"
echo "done $TAG"
