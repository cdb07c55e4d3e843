# c4 item search under the L2 hint: index+sector vs whole-node level 7, work-item size; c3 key-line evict-last repeat
mkdir -p gpurun_out
bash tools/sweep_cfg.sh s5c "c4" "" "--l2-levels 1099511627776" "--param item_rounds=8" "--param item_rounds=32"
bash tools/sweep_cfg.sh s5c "c3" "" "--param regular_l2_hint=2" "" "--param regular_l2_hint=2"
timeout 600 python bench.py > gpurun_out/s5c_bench_default.jsonl 2> gpurun_out/s5c_bench_default.err
