cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
GG_FORCE_DEVICE=0 GG_DIST_BACKEND=gloo timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29511 bench.py --gpus 2 --workload c5 --no-e2e > gpurun_out/c5_2rank.json 2> gpurun_out/c5_2rank.err
echo rc=$? >> gpurun_out/c5_2rank.err
