#!/bin/bash
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_bucketed.py tests/test_gpu_c4_full.py -x -q > gpurun_out/r02g23_tests.log 2>&1
echo "rc=$?" >> gpurun_out/r02g23_tests.log
timeout 900 python tools/param_sweep.py --config c4 --steps 10 --set item_first_sector=0 --set item_first_sector=1 --set item_first_sector=0 --set item_first_sector=1 --set item_first_sector=0 --set item_first_sector=1 > gpurun_out/r02g23_sweep.jsonl 2> gpurun_out/r02g23_sweep.err
