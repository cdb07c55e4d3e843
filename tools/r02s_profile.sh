#!/bin/bash
# Round-2 final profile set (TAG, default r02s): GPU tests, smoke, every 1-GPU
# config line, the c4 2-rank dry run, the default bench's launch list, single-pass
# steady-state DRAM traffic of each config's dominant kernel (-> profiles/traffic.json),
# and ncu --set full of the c4 item search.
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
TAG=${1:-r02s}
timeout 2400 python -m pytest tests -x -q -m gpu > gpurun_out/${TAG}_pytest_gpu.log 2>&1
echo "rc=$?" >> gpurun_out/${TAG}_pytest_gpu.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${TAG}_smoke.log 2>&1
# (compute-sanitizer is closed on this GPU pool since round 2b: tools/sanitize.sh, logs profiles/r02_sanitize_*)
for spec in "c2 implicit_search" "c1 implicit_search" "c5 implicit_search" "c3 regular_search_(items|cdir)" "c4 implicit_search_(items|cdir)"; do
  set -- $spec
  timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct,gpu__time_duration.sum \
    --cache-control none --clock-control none -k "regex:$2" -s 6 -c 2 --csv \
    python bench.py --config $1 --steps 8 --warmup 4 --no-cpu-baseline --e2e-steps 1 > gpurun_out/steady_$1.csv 2>&1
done
python tools/traffic_json.py gpurun_out $TAG > gpurun_out/${TAG}_traffic.log 2>&1
for c in c1 c2 c3 c5; do
  timeout 900 python bench.py --config $c --steps 50 --warmup 5 > gpurun_out/${TAG}_bench_$c.log 2>&1
done
timeout 900 python bench.py --steps 20 --warmup 5 > gpurun_out/${TAG}_bench_c4.log 2>&1
timeout 900 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/${TAG}_bench_reference.log 2>&1
timeout 900 python bench.py --gpus 2 --steps 10 --warmup 3 > gpurun_out/${TAG}_bench_c4_g2_one_gpu.log 2>&1
timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none -c 600 --csv \
  --log-file gpurun_out/${TAG}_launches_bench_default.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --e2e-steps 1 \
  > gpurun_out/${TAG}_launches_bench.log 2>&1
bash tools/ncu_c4_full.sh $TAG
