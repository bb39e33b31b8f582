#!/bin/bash
# The N > 1 bench path on a one-GPU box: two and three ranks on cuda:0 over gloo (host-staged
# collectives), default config 3 and the strong-scaling config-5 shard; then one NCCL rank.
set -u
TAG=${1:-r02p}
O=gpurun_out
mkdir -p $O
for N in 2 3; do
  timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node $N --master-addr 127.0.0.1 --master-port 29531 \
    bench.py --gpus $N --steps 3 --warmup 3 --backend gloo --one-device --no-configs --nseq 100000 > $O/bench_n${N}_$TAG.json 2> $O/bench_n${N}_$TAG.err
  echo "N=$N rc=$?" >> $O/bench_multi_$TAG.log
done
timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29532 \
  bench.py --gpus 2 --steps 3 --warmup 3 --backend gloo --one-device --config 5 --which 0 --nseq 400000 > $O/bench_n2c5_$TAG.json 2> $O/bench_n2c5_$TAG.err
echo "c5 rc=$?" >> $O/bench_multi_$TAG.log
timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 --master-port 29533 \
  bench.py --gpus 1 --steps 3 --warmup 3 --no-configs --no-cpu-baseline > $O/bench_n1tr_$TAG.json 2> $O/bench_n1tr_$TAG.err
echo "torchrun n1 rc=$?" >> $O/bench_multi_$TAG.log
timeout 600 python bench.py --impl reference --steps 2 --warmup 3 > $O/bench_ref_$TAG.json 2> $O/bench_ref_$TAG.err
echo "ref rc=$?" >> $O/bench_multi_$TAG.log
echo done
