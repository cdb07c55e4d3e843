#!/bin/bash
# ncu --set full of the c4 partition kernels (count, scatter, gather) -- one steady launch each
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
for K in bk_count bk_scatter bk_gather_rec; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:$K -s 3 -c 1 \
    -o gpurun_out/r02g9_$K python tools/param_sweep.py --config c4 --steps 1 --set item_sched=0 > gpurun_out/r02g9_$K.log 2>&1
done
