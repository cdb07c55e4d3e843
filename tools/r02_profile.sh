#!/bin/bash
# round-2 profile set: every 1-GPU config line, the default bench's launch list, single-pass
# steady-state DRAM traffic per config, and ncu --set full of the c4 item search.
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
TAG=${1:-r02}
timeout 2400 python -m pytest tests -x -q -m gpu > gpurun_out/${TAG}_pytest_gpu.log 2>&1
echo "rc=$?" >> gpurun_out/${TAG}_pytest_gpu.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${TAG}_smoke.log 2>&1
bash tools/sanitize.sh
for c in c1 c2 c3 c5; do
  timeout 900 python bench.py --config $c --steps 50 --warmup 5 > gpurun_out/${TAG}_bench_$c.log 2>&1
done
timeout 900 python bench.py --steps 20 --warmup 5 > gpurun_out/${TAG}_bench_c4.log 2>&1
timeout 900 python bench.py --gpus 2 --steps 10 --warmup 3 > gpurun_out/${TAG}_bench_c4_g2_one_gpu.log 2>&1
# launch list of the default command (times are cold-cache and serialised: compare shares)
timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none -c 600 --csv \
  --log-file gpurun_out/${TAG}_launches_bench_default.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --e2e-steps 1 \
  > gpurun_out/${TAG}_launches_bench.log 2>&1
# single-pass DRAM bytes of each config's dominant kernel, steady state
for spec in "c2 implicit_search" "c1 implicit_search" "c5 implicit_search" "c3 regular_search_(items|cdir)" "c4 implicit_search_(items|cdir)"; do
  set -- $spec
  timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct,gpu__time_duration.sum \
    --cache-control none --clock-control none -k "regex:$2" -s 6 -c 2 --csv \
    python bench.py --config $1 --steps 8 --warmup 4 --no-cpu-baseline --e2e-steps 1 > gpurun_out/steady_$1.csv 2>&1
done
# the top kernel, full set (c4 item search, one steady launch)
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"implicit_search_(items|cdir)" -s 3 -c 1 \
  -o gpurun_out/${TAG}_c4_items_full python tools/param_sweep.py --config c4 --steps 1 > gpurun_out/${TAG}_c4_items_full.log 2>&1
