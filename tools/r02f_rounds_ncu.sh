cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
for r in 16 8 4; do
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct,smsp__average_warps_issue_stalled_barrier_per_issue_active.ratio,smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio,l1tex__data_pipe_lsu_wavefronts.avg.pct_of_peak_sustained_elapsed \
  --cache-control none --clock-control none -k regex:implicit_search_items -s 3 -c 1 --csv \
  python tools/param_sweep.py --config c4 --steps 3 --set item_rounds=$r > gpurun_out/r02f_rounds_$r.csv 2>&1
done
