# single-pass (no replay) DRAM bytes per launch of the search kernel, steady state, per config
for spec in "c2 implicit_search" "c1 implicit_search" "c5 implicit_search" "c3 regular_search_items" "c4 implicit_search"; do
  set -- $spec
  timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct,gpu__time_duration.sum \
    --cache-control none --clock-control none -k regex:$2 -s 6 -c 2 --csv \
    python bench.py --config $1 --steps 8 --warmup 4 --no-cpu-baseline --e2e-steps 1 > gpurun_out/steady_$1.csv 2>&1
done
