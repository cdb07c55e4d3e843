#!/bin/bash
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 900 python tools/param_sweep.py --config c4 --steps 5 --set item_cap_slack=0 --set item_cap_slack=1 --set item_cap_slack=2 --set item_cap_slack=4 --set item_cap_slack=1,item_rounds=32 --set item_cap_slack=1,item_rounds=8 > gpurun_out/r02g12_sweep.jsonl 2> gpurun_out/r02g12_sweep.err
timeout 900 python tools/param_sweep.py --config c3 --steps 10 --set item_cap_slack=0 --set item_cap_slack=1 --set item_cap_slack=2 --set item_cap_slack=4 >> gpurun_out/r02g12_sweep.jsonl 2>> gpurun_out/r02g12_sweep.err
