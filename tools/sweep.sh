# usage: bash tools/sweep.sh <tag> "<args1>" "<args2>" ...
tag=$1; shift
for cfg in "$@"; do
  timeout 300 python bench.py --steps 200 --warmup 5 --no-cpu-baseline --e2e-steps 1 $cfg > gpurun_out/sweep_${tag}.tmp 2>&1
  echo "== $cfg" >> gpurun_out/sweep_${tag}.log
  tail -1 gpurun_out/sweep_${tag}.tmp >> gpurun_out/sweep_${tag}.log
done
rm -f gpurun_out/sweep_${tag}.tmp
