#!/bin/bash
# GPU session: the bench's multi-rank paths as 2 ranks sharing one GPU (gloo) (tool).
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
for wl in c2 c5; do
  GG_FORCE_DEVICE=0 GG_DIST_BACKEND=gloo timeout 1200 python -m torch.distributed.run --nnodes=1 \
    --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 2951$([ $wl = c2 ] && echo 1 || echo 2) \
    bench.py --gpus 2 --workload $wl --steps 2 > gpurun_out/mr_$wl.json 2> gpurun_out/mr_$wl.err
  echo "rc=$?" >> gpurun_out/mr_$wl.err
done
