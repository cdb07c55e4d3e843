# Session-5 evidence with the L2-hint defaults: steady DRAM traffic per config, the ncu
# launch list of the default bench command, full captures of the c2 search and the c4
# item search (summarised on the box; the .ncu-rep files stay in gpurun_out/)
tag=${1:-r01s5}
mkdir -p gpurun_out
bash tools/steady_traffic.sh
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 600 --csv \
  --log-file gpurun_out/${tag}_launches_bench_default.csv python bench.py --steps 20 --warmup 3 --no-cpu-baseline \
  > gpurun_out/${tag}_launches_bench.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:implicit_search -s 10 -c 1 \
  -o gpurun_out/${tag}_c2_full python bench.py --steps 20 --warmup 3 --no-cpu-baseline --e2e-steps 1 \
  > gpurun_out/${tag}_c2_full.log 2>&1
python tools/ncu_summary.py gpurun_out/${tag}_c2_full.ncu-rep > gpurun_out/${tag}_c2_ncu_summary.txt 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:search_items -s 4 -c 1 \
  -o gpurun_out/${tag}_c4_items_full python bench.py --config c4 --steps 5 --warmup 3 --no-cpu-baseline --e2e-steps 1 \
  > gpurun_out/${tag}_c4_full.log 2>&1
python tools/ncu_summary.py gpurun_out/${tag}_c4_items_full.ncu-rep > gpurun_out/${tag}_c4_items_ncu_summary.txt 2>&1
echo done
