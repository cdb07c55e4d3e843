# A/B ncu counters per design lever (SURVEY 8(d) "Evidence per design lever"): one
# steady-state launch of the dominant kernel per variant, a fixed metric list.
# Output: gpurun_out/ab_<tag>.csv per variant; tools/lever_table.py summarises.
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct,\
lts__t_sectors_srcunit_tex_op_read.sum,l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum,\
l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum,l1tex__data_pipe_lsu_wavefronts.avg.pct_of_peak_sustained_elapsed,\
l1tex__t_sector_hit_rate.pct,smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio,\
dram__throughput.avg.pct_of_peak_sustained_elapsed,l1tex__data_pipe_lsu_wavefronts_mem_shared.sum
run() {  # tag kernel-regex bench-args...
  tag=$1; kre=$2; shift; shift
  timeout 900 ncu --metrics $M --cache-control none --clock-control none --print-units base -k regex:$kre -s 6 -c 1 --csv \
    python bench.py --steps 8 --warmup 4 --no-cpu-baseline --e2e-steps 1 --graph 0 "$@" > gpurun_out/ab_${tag}.csv 2>&1
}
run c2_default implicit_search --config c2
run c2_leaf16 implicit_search --config c2 --leaf256 0
run c2_staged_levels implicit_search --config c2 --smem-mode 0
run c2_whole_nodes implicit_search --config c2 --full-levels 48
run c5_default implicit_search --config c5
run c5_full16 implicit_search --config c5 --param full256=0
run c3_bucketed regular_search_items --config c3
run c3_unbucketed regular_search_v2 --config c3 --bucket 0
echo done
