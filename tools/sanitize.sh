#!/bin/bash
# compute-sanitizer runs over tools/sanitize_scenarios.py (every kernel family on tiny
# inputs, results checked against the oracle) and the two-process fused exchange.
# Logs: gpurun_out/sanitize_<tool>.log (copied to profiles/ by hand).
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
CS=/usr/local/cuda/bin/compute-sanitizer
for tool in memcheck racecheck synccheck initcheck; do
  timeout 1500 $CS --tool $tool --error-exitcode 9 --print-limit 50 --kernel-name-exclude kns=at6native \
    python tools/sanitize_scenarios.py > gpurun_out/sanitize_$tool.log 2>&1
  echo "exit=$?" >> gpurun_out/sanitize_$tool.log
done
# two processes on one GPU: CUDA IPC windows, device barriers, peer stores
PORT=$((20000 + RANDOM % 20000))
timeout 1200 $CS --tool memcheck --target-processes all --error-exitcode 9 --print-limit 50 \
  python -m torch.distributed.run --nproc-per-node 2 --master-addr 127.0.0.1 --master-port $PORT \
  tools/two_rank_one_gpu.py 0 1 > gpurun_out/sanitize_memcheck_two_process.log 2>&1
echo "exit=$?" >> gpurun_out/sanitize_memcheck_two_process.log
