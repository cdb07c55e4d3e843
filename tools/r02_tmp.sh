#!/bin/bash
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_bucketed.py tests/test_gpu_placement.py -x -q > gpurun_out/r02g22_tests.log 2>&1
echo "rc=$?" >> gpurun_out/r02g22_tests.log
timeout 900 python tools/param_sweep.py --config c4 --steps 5 --set gather_tma=0 --set gather_tma=1 --set gather_tma=0 --set gather_tma=1 > gpurun_out/r02g22_sweep.jsonl 2> gpurun_out/r02g22_sweep.err
timeout 900 python tools/param_sweep.py --config c3 --steps 10 --set gather_tma=0 --set gather_tma=1 >> gpurun_out/r02g22_sweep.jsonl 2>> gpurun_out/r02g22_sweep.err
