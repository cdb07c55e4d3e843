cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 900 python tools/param_sweep.py --config c4 --steps 10 --set item_dir32=1 --set item_rounds=4 --set item_rounds=0 > gpurun_out/r02g_unsorted.jsonl 2>&1
timeout 900 python tools/param_sweep.py --config c4 --steps 10 --sorted --set item_dir32=1 --set item_rounds=4 --set item_rounds=0 > gpurun_out/r02g_sorted.jsonl 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,lts__t_sector_hit_rate.pct \
  --cache-control none --clock-control none -k regex:implicit_search_items -s 3 -c 1 --csv \
  python tools/param_sweep.py --config c4 --steps 3 --sorted > gpurun_out/r02g_sorted_ncu.csv 2>&1
