#!/bin/bash
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_bucketed.py tests/test_gpu_c4_full.py tests/test_gpu_placement.py tests/test_gpu_sharded.py -x -q > gpurun_out/r02g24_tests.log 2>&1
echo "rc=$?" >> gpurun_out/r02g24_tests.log
timeout 900 python tools/param_sweep.py --config c4 --steps 10 --set scatter_tma=0 --set scatter_tma=1 --set scatter_tma=0 --set scatter_tma=1 > gpurun_out/r02g24_sweep.jsonl 2> gpurun_out/r02g24_sweep.err
