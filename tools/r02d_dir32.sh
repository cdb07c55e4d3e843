#!/bin/bash
# compressed item directory: bucketed parity suite, c4 / c5 A/B (item_dir32 0 vs 1), item size sweep
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
TAG=${1:-r02d}
timeout 900 python -m pytest tests/test_gpu_bucketed.py tests/test_gpu_c4_full.py -x -q > gpurun_out/${TAG}_bucketed.log 2>&1; echo "rc=$?" >> gpurun_out/${TAG}_bucketed.log
timeout 900 python tools/param_sweep.py --config c4 --steps 10 --set item_dir32=0 --set item_dir32=1 --set item_dir32=0 --set item_dir32=1 \
  --set item_rounds=8 --set item_rounds=4 --set item_rounds=2 --set item_rounds=0 > gpurun_out/${TAG}_c4_dir32.jsonl 2>&1
timeout 600 python tools/param_sweep.py --config c5 --steps 20 --set item_dir32=0 --set item_dir32=1 --set item_dir32=0 --set item_dir32=1 \
  --set item_rounds=8 --set item_rounds=4 --set item_rounds=0 > gpurun_out/${TAG}_c5_dir32.jsonl 2>&1
