#!/bin/bash
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 900 python tools/param_sweep.py --config c5 --steps 10 --set bucket=0 --set bucket=1 --set bucket=1,bucket_slice=4194304 --set bucket=0 > gpurun_out/r02g25_sweep.jsonl 2> gpurun_out/r02g25_sweep.err
timeout 900 python tools/param_sweep.py --config c2 --steps 20 --set bucket=0 --set bucket=1 >> gpurun_out/r02g25_sweep.jsonl 2>> gpurun_out/r02g25_sweep.err
