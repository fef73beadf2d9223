cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
for rep in 1 2; do for t in 16 12 8 6; do
  echo "threads $t" >> gpurun_out/lr_ab.txt
  HOST_THREADS=$t REPS=3 timeout 300 python tools/lr_trace.py 2>&1 | grep "wall ms" | cut -c1-40 >> gpurun_out/lr_ab.txt
done; done
