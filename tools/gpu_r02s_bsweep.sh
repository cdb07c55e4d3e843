#!/bin/bash
# bucket-count sweeps (bucket_slice) for the bucketed configs with the compressed directory
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 900 python tools/param_sweep.py --config c4 --steps 10 --set bucket_slice=52000000 --set bucket_slice=55000000 \
  --set bucket_slice=58000000 --set bucket_slice=61000000 --set bucket_slice=64000000 --set bucket_slice=68000000 \
  --set bucket_slice=0 --set bucket_slice=58000000 --set bucket_slice=64000000 > gpurun_out/r02s_c4_bucket_sweep2.jsonl 2>&1
timeout 600 python tools/param_sweep.py --config c5 --steps 20 --set bucket_slice=0 --set bucket_slice=3000000 \
  --set bucket_slice=3500000 --set bucket_slice=4000000 --set bucket_slice=0 > gpurun_out/r02s_c5_bucket_sweep.jsonl 2>&1
timeout 600 python tools/param_sweep.py --config c3 --steps 20 --set bucket_slice=0 --set bucket_slice=3000000 \
  --set bucket_slice=3300000 --set bucket_slice=0 > gpurun_out/r02s_c3_bucket_sweep.jsonl 2>&1
