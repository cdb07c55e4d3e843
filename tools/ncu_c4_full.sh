#!/bin/bash
# ncu --set full of one steady c4 item-search launch, exported as raw + source CSV here on the box.
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
TAG=${1:-r02s}; shift
timeout 1500 ncu --set full --clock-control none --import-source on -k "regex:implicit_search_(items|cdir)" -s 3 -c 1 \
  -o gpurun_out/${TAG}_c4_items_full python tools/param_sweep.py --config c4 --steps 1 "$@" > gpurun_out/${TAG}_c4_items_full.log 2>&1
ncu -i gpurun_out/${TAG}_c4_items_full.ncu-rep --page raw --csv > gpurun_out/${TAG}_c4_items_raw.csv 2>&1
ncu -i gpurun_out/${TAG}_c4_items_full.ncu-rep --page source --csv --print-source sass > gpurun_out/${TAG}_c4_items_sass.csv 2>&1
ncu -i gpurun_out/${TAG}_c4_items_full.ncu-rep --page details --csv > gpurun_out/${TAG}_c4_items_details.csv 2>&1
