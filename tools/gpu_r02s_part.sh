#!/bin/bash
# c4 bucket-count sweep with the compressed directory, and ncu --set full of the partition kernels.
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 900 python tools/param_sweep.py --config c4 --steps 10 --set bucket_slice=0 --set bucket_slice=47000000 \
  --set bucket_slice=58000000 --set bucket_slice=76000000 --set bucket_slice=0 --set bucket_slice=76000000 \
  > gpurun_out/r02s_c4_bucket_sweep.jsonl 2>&1
for k in bk_gather_rec bk_scatter_tma bk_count; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:"$k" -s 2 -c 1 \
    -o gpurun_out/r02s_c4_$k python tools/param_sweep.py --config c4 --steps 1 > gpurun_out/r02s_c4_$k.log 2>&1
  ncu -i gpurun_out/r02s_c4_$k.ncu-rep --page raw --csv > gpurun_out/r02s_c4_${k}_raw.csv 2>&1
  ncu -i gpurun_out/r02s_c4_$k.ncu-rep --page source --csv --print-source sass > gpurun_out/r02s_c4_${k}_sass.csv 2>&1
done
