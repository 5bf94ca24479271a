#!/bin/bash
# Multi-process bench path on a one-GPU box: (1) the sharded pipeline as a one-rank NCCL group,
# (2) two ranks sharing the GPU over gloo (host-staged collectives) -- exercises torchrun, the
# partition / exchange / merge orchestration and max-over-ranks timing end to end.
timeout 600 python bench.py --config C5 --events 1000000000 --steps 3 --sharded --no-cpu-baseline --e2e-steps 1 \
  > gpurun_out/r01s4_sharded_n1.json 2> gpurun_out/r01s4_sharded_n1.err; echo "n1 rc=$?"
timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 \
  bench.py --gpus 2 --backend gloo --config C5 --events 500000000 --steps 3 --no-cpu-baseline --e2e-steps 1 \
  > gpurun_out/r01s4_gloo_n2.json 2> gpurun_out/r01s4_gloo_n2.err; echo "n2 rc=$?"
