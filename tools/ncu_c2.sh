# full ncu capture of the c2 search kernel; $1 = tag, rest = extra bench args
tag=$1; shift
timeout 600 ncu --set full --clock-control none --import-source on -k regex:implicit_search -s 3 -c 1 \
  -o gpurun_out/prof_${tag} python bench.py --steps 2 --warmup 3 --no-cpu-baseline --e2e-steps 1 "$@" > gpurun_out/ncu_${tag}.log 2>&1
timeout 600 ncu --set full --cache-control none --clock-control none -k regex:implicit_search -s 3 -c 1 \
  -o gpurun_out/prof_${tag}_warm python bench.py --steps 2 --warmup 3 --no-cpu-baseline --e2e-steps 1 "$@" > gpurun_out/ncu_${tag}_warm.log 2>&1
