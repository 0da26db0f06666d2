#!/bin/bash
# the N>1 bench path as 2 processes sharing one GPU (gloo process group;
# the driver's multi-GPU runs use NCCL on separate GPUs)
mkdir -p gpurun_out
for ex in nccl fused; do
  timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29511 \
    bench.py --gpus 2 --dist-backend gloo --exchange $ex --config cfg3b --steps 5 --warmup 3 --no-cpu-baseline \
    > gpurun_out/multirank_$ex.json 2> gpurun_out/multirank_$ex.log
  echo "exit $?" >> gpurun_out/multirank_$ex.log
done
