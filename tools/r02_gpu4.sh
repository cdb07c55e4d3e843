#!/bin/bash
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 1200 python tools/param_sweep.py --config c4 --steps 5 \
  --set item_sched=0,bucket_slice=0 --set item_sched=0,bucket_slice=41943040 \
  --set item_sched=0,bucket_slice=75497472 --set item_sched=0,bucket_slice=150994944 \
  --set item_sched=0,bucket_slice=301989888 > gpurun_out/r02g4_sweep.jsonl 2> gpurun_out/r02g4_sweep.err
