#!/bin/bash
# ncu A/B of the c4 implicit item search: contiguous (item_sched=0) vs strided (1) items
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
M="gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct,lts__t_sectors_srcunit_tex_op_read.sum,sm__warps_active.avg.pct_of_peak_sustained_active,l1tex__data_pipe_lsu_wavefronts.avg.pct_of_peak_sustained_elapsed,l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared.sum,smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio,smsp__inst_executed.sum,launch__shared_mem_per_block_dynamic,l1tex__t_sector_hit_rate.pct"
for S in "item_sched=0,item_l2_hint=1" "item_sched=1,item_l2_hint=1" "item_sched=1,item_l2_hint=0"; do
  tag=$(echo $S | tr ',=' '__')
  timeout 900 ncu --metrics $M --clock-control none -k regex:implicit_search_items -s 3 -c 1 --csv \
    --log-file gpurun_out/r02g6_$tag.csv python tools/param_sweep.py --config c4 --steps 1 --set $S > gpurun_out/r02g6_$tag.log 2>&1
done
