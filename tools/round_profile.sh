# Round-end evidence on one GPU: default bench line, reference arm, the ncu
# launch list of the bench command, and one full capture of the top kernel.
# $1 = round tag (e.g. r01)
tag=${1:-r01}
mkdir -p gpurun_out
timeout 600 python bench.py > gpurun_out/${tag}_bench_default.jsonl 2> gpurun_out/${tag}_bench_default.err
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/${tag}_bench_reference.jsonl 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 600 --csv \
  --log-file gpurun_out/${tag}_launches_bench_default.csv python bench.py --steps 20 --warmup 3 --no-cpu-baseline \
  > gpurun_out/${tag}_launches_bench.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:implicit_search -s 10 -c 1 \
  -o gpurun_out/${tag}_c2_full python bench.py --steps 20 --warmup 3 --no-cpu-baseline --e2e-steps 1 \
  > gpurun_out/${tag}_c2_full.log 2>&1
echo done
