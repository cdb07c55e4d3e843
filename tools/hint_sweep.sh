# L2 eviction-priority hint A/B (l2_hint / item_l2_hint knobs): bench lines + single-pass DRAM traffic
mkdir -p gpurun_out
bash tools/sweep_cfg.sh hint c4 "" "--param item_l2_hint=1" "--param item_l2_hint=2" "--param item_l2_hint=3"
bash tools/sweep_cfg.sh hint c5 "" "--param l2_hint=1" "--param l2_hint=2" "--param l2_hint=3"
bash tools/sweep_cfg.sh hint c2 "" "--param l2_hint=1" "--param l2_hint=2"
for h in 0 1 3; do
  timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct,gpu__time_duration.sum \
    --cache-control none --clock-control none -k regex:implicit_search -s 6 -c 2 --csv \
    python bench.py --config c4 --steps 8 --warmup 4 --no-cpu-baseline --e2e-steps 1 --param item_l2_hint=$h > gpurun_out/hint_steady_c4_$h.csv 2>&1
done
