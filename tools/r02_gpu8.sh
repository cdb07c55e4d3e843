#!/bin/bash
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_concurrency.py -x -q -s > gpurun_out/r02g8_conc.log 2>&1
echo "rc=$?" >> gpurun_out/r02g8_conc.log
timeout 1500 python -m pytest tests -x -q -m gpu -k "not c4_full and not c3_full and not concurrency" > gpurun_out/r02g8_gpu.log 2>&1
echo "rc=$?" >> gpurun_out/r02g8_gpu.log
