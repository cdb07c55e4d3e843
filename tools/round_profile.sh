# Round-end evidence on one GPU: default bench line, reference arm, the other 1-GPU
# configs, the ncu launch list of the bench command, full captures of the dominant
# kernels (c2 search, c3 bucketed item search) and steady-state DRAM traffic per config.
# $1 = round tag (e.g. r01)
tag=${1:-r01}
mkdir -p gpurun_out
timeout 600 python bench.py > gpurun_out/${tag}_bench_default.jsonl 2> gpurun_out/${tag}_bench_default.err
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/${tag}_bench_reference.jsonl 2>&1
: > gpurun_out/${tag}_configs_1gpu.jsonl
for c in c1 c3 c5 c4; do
  timeout 900 python bench.py --config $c --steps 50 --warmup 5 > gpurun_out/bench_$c.log 2>&1
  tail -1 gpurun_out/bench_$c.log >> gpurun_out/${tag}_configs_1gpu.jsonl
done
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 600 --csv \
  --log-file gpurun_out/${tag}_launches_bench_default.csv python bench.py --steps 20 --warmup 3 --no-cpu-baseline \
  > gpurun_out/${tag}_launches_bench.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"bk_|search|DeviceScan" -c 200 --csv \
  --log-file gpurun_out/${tag}_launches_bench_c3.csv python bench.py --config c3 --steps 5 --warmup 3 --no-cpu-baseline \
  --e2e-steps 1 > gpurun_out/${tag}_launches_c3.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:implicit_search -s 10 -c 1 \
  -o gpurun_out/${tag}_c2_full python bench.py --steps 20 --warmup 3 --no-cpu-baseline --e2e-steps 1 \
  > gpurun_out/${tag}_c2_full.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:search_items -s 4 -c 1 \
  -o gpurun_out/${tag}_c3_items_full python bench.py --config c3 --steps 5 --warmup 3 --no-cpu-baseline --e2e-steps 1 \
  > gpurun_out/${tag}_c3_full.log 2>&1
bash tools/steady_traffic.sh
echo done
