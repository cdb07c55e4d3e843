# full ncu capture of the search kernel of one config; $1 = tag, $2 = kernel regex, rest = bench args
tag=$1; kre=$2; shift; shift
timeout 900 ncu --set full --clock-control none --import-source on -k regex:$kre -s 3 -c 1 \
  -o gpurun_out/prof_${tag} python bench.py --steps 2 --warmup 3 --no-cpu-baseline --e2e-steps 1 "$@" > gpurun_out/ncu_${tag}.log 2>&1
timeout 600 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct,gpu__time_duration.sum \
  --cache-control none --clock-control none -k regex:$kre -s 6 -c 2 --csv python bench.py --steps 8 --warmup 4 \
  --no-cpu-baseline --e2e-steps 1 "$@" > gpurun_out/ncu_${tag}_steady.csv 2>&1
