#!/bin/bash
# bench.py's N>1 path (torchrun, NCCL) with both ranks on the one sandbox GPU
# (CUALIGN_ONE_GPU=1): checks the contract end to end; not a B200 scaling number.
set -u
OUT=gpurun_out/${1:-n2}
mkdir -p $OUT
export CUALIGN_ONE_GPU=1
timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 \
   bench.py --gpus 2 --steps 20 --warmup 3 > $OUT/bench_n2.json 2> $OUT/bench_n2.err; echo "n2 rc=$?"; tail -1 $OUT/bench_n2.json | cut -c1-1500
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29534 \
   bench.py --impl reference --gpus 2 --steps 3 --warmup 3 > $OUT/ref_n2.json 2> $OUT/ref_n2.err; echo "ref rc=$?"; tail -1 $OUT/ref_n2.json | cut -c1-800
