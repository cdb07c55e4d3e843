#!/bin/bash
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_bucketed.py tests/test_gpu_sharded.py tests/test_gpu_placement.py -x -q > gpurun_out/r02g13_tests.log 2>&1
echo "rc=$?" >> gpurun_out/r02g13_tests.log
timeout 900 python tools/param_sweep.py --config c4 --steps 5 --set partition_direct=0 --set partition_direct=1 --set partition_direct=0 --set partition_direct=1 > gpurun_out/r02g13_sweep.jsonl 2> gpurun_out/r02g13_sweep.err
timeout 900 python tools/param_sweep.py --config c3 --steps 10 --set partition_direct=0 --set partition_direct=1 >> gpurun_out/r02g13_sweep.jsonl 2>> gpurun_out/r02g13_sweep.err
