#!/bin/bash
# ncu --set full of one steady c4 item-search launch: tools/ncu_items.sh TAG [param_sweep --set ...]
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
TAG=$1; shift
timeout 1200 ncu --set full --clock-control none --import-source on -k "regex:implicit_search_(items|cdir)" -s 3 -c 1 \
  -o gpurun_out/${TAG}_c4_items_full python tools/param_sweep.py --config c4 --steps 1 "$@" > gpurun_out/${TAG}_c4_items_full.log 2>&1
