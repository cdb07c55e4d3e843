#!/bin/bash
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_bucketed.py tests/test_gpu_c4_full.py -x -q -m gpu > gpurun_out/r02s_pytest_scatter.log 2>&1; echo "rc=$?" >> gpurun_out/r02s_pytest_scatter.log
timeout 600 python tools/param_sweep.py --config c4 --steps 10 --set scatter_wcoop=0 --set scatter_wcoop=1 --set scatter_wcoop=0 --set scatter_wcoop=1 > gpurun_out/r02s_c4_scatter_ab.jsonl 2>&1
timeout 600 python tools/param_sweep.py --config c3 --steps 20 --set scatter_wcoop=0 --set scatter_wcoop=1 --set scatter_wcoop=0 --set scatter_wcoop=1 >> gpurun_out/r02s_c4_scatter_ab.jsonl 2>&1
