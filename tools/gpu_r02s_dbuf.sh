#!/bin/bash
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_bucketed.py tests/test_gpu_c4_full.py -x -q -m gpu > gpurun_out/r02s_pytest_dbuf.log 2>&1; echo "rc=$?" >> gpurun_out/r02s_pytest_dbuf.log
timeout 900 python tools/param_sweep.py --config c4 --steps 10 --set item_dbuf=0,item_rounds=16 --set item_dbuf=0,item_rounds=8 \
  --set item_dbuf=1,item_rounds=8 --set item_dbuf=1,item_rounds=4 --set item_dbuf=1,item_rounds=2 --set item_dbuf=1,item_rounds=16 \
  --set item_dbuf=0,item_rounds=8 --set item_dbuf=1,item_rounds=4 --set item_dbuf=1,item_rounds=8 > gpurun_out/r02s_c4_dbuf_sweep.jsonl 2>&1
timeout 900 python tools/param_sweep.py --config c5 --steps 20 --set item_dbuf=0,item_rounds=16 --set item_dbuf=0,item_rounds=8 \
  --set item_dbuf=1,item_rounds=8 --set item_dbuf=1,item_rounds=4 --set item_dbuf=1,item_rounds=2 --set item_dbuf=0,item_rounds=16 > gpurun_out/r02s_c5_dbuf_sweep.jsonl 2>&1
