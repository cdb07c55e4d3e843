#!/bin/bash
# direct gather: bucketed parity suites, then A/B against the staged gather on c4 / c3 / c5
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_bucketed.py tests/test_gpu_c4_full.py tests/test_gpu_sharded.py -x -q -m gpu > gpurun_out/r02s_pytest_gather.log 2>&1; echo "rc=$?" >> gpurun_out/r02s_pytest_gather.log
timeout 600 python tools/param_sweep.py --config c4 --steps 10 --set gather_direct=0 --set gather_direct=1 --set gather_direct=0 --set gather_direct=1 > gpurun_out/r02s_c4_gather_ab.jsonl 2>&1
timeout 600 python tools/param_sweep.py --config c3 --steps 20 --set gather_direct=0 --set gather_direct=1 --set gather_direct=0 --set gather_direct=1 > gpurun_out/r02s_c3_gather_ab.jsonl 2>&1
timeout 600 python tools/param_sweep.py --config c5 --steps 20 --set gather_direct=0 --set gather_direct=1 --set gather_direct=0 --set gather_direct=1 > gpurun_out/r02s_c5_gather_ab.jsonl 2>&1
