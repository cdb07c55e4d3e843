#!/bin/bash
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_sharded.py tests/test_gpu_bucketed.py tests/test_gpu_placement.py tests/test_gpu_c4_full.py tests/test_gpu_concurrency.py -x -q > gpurun_out/r02g10_tests.log 2>&1
echo "rc=$?" >> gpurun_out/r02g10_tests.log
timeout 900 python tools/param_sweep.py --config c4 --steps 5 --set item_sched=0 > gpurun_out/r02g10_sweep.jsonl 2> gpurun_out/r02g10_sweep.err
timeout 900 python tools/param_sweep.py --config c3 --steps 10 --set bucket=2 >> gpurun_out/r02g10_sweep.jsonl 2>> gpurun_out/r02g10_sweep.err
