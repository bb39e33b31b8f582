#!/bin/bash
# Forward: one-warp geometries with 12 / 13 / 14 nodes per thread (M = 257 ... 448; config 3's M = 400
# at 13 instead of 16): Forward parity (tolerance), then the bench forward leg vs FWD_QMAX=8 / the
# 16-node geometry (tools/fwd_bench.py style via the bench leg)
set -u
TAG=${1:-r02zzo}
O=gpurun_out
mkdir -p $O
timeout 1800 python -m pytest tests/test_gpu_forward.py -q -x > $O/tests_fwd_$TAG.log 2>&1
timeout 600 python bench.py --batch 0 --steps 5 --no-cpu-baseline --no-e2e --no-configs > $O/bench_fwd_$TAG.json 2> $O/bench_fwd_$TAG.err
HMG_NVCC_EXTRA=-DFWD_NO_Q13 python -c "from paper_conf_ipps_jiangg15_b200 import build; build.build(force=True)"
timeout 600 python bench.py --batch 0 --steps 5 --no-cpu-baseline --no-e2e --no-configs > $O/bench_fwd16_$TAG.json 2> $O/bench_fwd16_$TAG.err
python -c "from paper_conf_ipps_jiangg15_b200 import build; build.build(force=True)"
echo "done $TAG"
