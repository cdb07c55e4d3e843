#!/bin/bash
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 1200 python tools/param_sweep.py --config c4 --steps 5 \
  --set item_sched=0,item_l2_hint=1 --set item_sched=1,item_l2_hint=0 --set item_sched=1,item_l2_hint=1 \
  --set item_sched=1,item_l2_hint=0,item_rounds=6 \
  > gpurun_out/r02g7_sweep.jsonl 2> gpurun_out/r02g7_sweep.err
