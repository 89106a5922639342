#!/bin/bash
# the N>1 bench flow (split row: local select + all-gather of packed candidates + merge) with two
# ranks sharing the one GPU over gloo (NCCL needs distinct GPUs): exercises bench.py's multi-rank path
mkdir -p gpurun_out
timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 \
  bench.py --gpus 2 --steps 5 --warmup 3 --dist-backend gloo --no-cpu --no-extras --e2e-steps 1 \
  > gpurun_out/multirank_c3.json 2> gpurun_out/multirank_c3.err
echo "c3 exit=$?" > gpurun_out/multirank_summary.txt
timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29534 \
  bench.py --gpus 2 --steps 5 --warmup 3 --config c2 --dist-backend gloo --no-cpu --no-extras --e2e-steps 1 \
  > gpurun_out/multirank_c2.json 2> gpurun_out/multirank_c2.err
echo "c2 exit=$?" >> gpurun_out/multirank_summary.txt
