#!/bin/bash
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_bucketed.py -x -q -k "not c3_full" > gpurun_out/r02g5_bucketed.log 2>&1
echo "rc=$?" >> gpurun_out/r02g5_bucketed.log
timeout 1200 python tools/param_sweep.py --config c4 --steps 5 \
  --set item_sched=0,item_rounds=0,item_l2_hint=1 \
  --set item_sched=1,item_rounds=0,item_l2_hint=1 --set item_sched=1,item_rounds=0,item_l2_hint=0 \
  --set item_sched=1,item_rounds=4,item_l2_hint=0 --set item_sched=1,item_rounds=2,item_l2_hint=0 \
  > gpurun_out/r02g5_sweep.jsonl 2> gpurun_out/r02g5_sweep.err
timeout 900 python -m pytest tests/test_gpu_c4_full.py -x -q > gpurun_out/r02g5_c4tests.log 2>&1
echo "rc=$?" >> gpurun_out/r02g5_c4tests.log
