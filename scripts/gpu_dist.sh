#!/bin/bash
# exercise bench.py's multi-rank path on one GPU (gloo control plane, all ranks on GPU 0)
mkdir -p gpurun_out
for n in 2 4; do
  BENCH_SAME_DEVICE=1 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node $n \
    --master-addr 127.0.0.1 --master-port 29511 bench.py --gpus $n --steps 5 --warmup 3 \
    --dist-backend gloo --no-cpu > gpurun_out/dist_$n.json 2> gpurun_out/dist_$n.err
  echo "exit $?" >> gpurun_out/dist_$n.err
done
BENCH_SAME_DEVICE=1 timeout 300 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 \
  --master-addr 127.0.0.1 --master-port 29512 bench.py --impl reference --gpus 2 --steps 2 --warmup 1 \
  > gpurun_out/dist_ref.json 2> gpurun_out/dist_ref.err
echo "exit $?" >> gpurun_out/dist_ref.err
