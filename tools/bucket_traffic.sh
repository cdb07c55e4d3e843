# Per-kernel device time and DRAM bytes of the bucketed pipeline (steady state, single pass).
mkdir -p gpurun_out
for spec in ${SPECS:-"c3 16777216" "c5 16777216"}; do
  set -- $spec
  timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct,gpu__time_duration.sum \
    --cache-control none --clock-control none -k regex:"bk_|search" -s 12 -c 10 --csv \
    python bench.py --config $1 --steps 6 --warmup 3 --no-cpu-baseline --e2e-steps 1 --bucket 1 --bucket-slice $2 \
    > gpurun_out/bt_$1_$2.csv 2>&1
done
