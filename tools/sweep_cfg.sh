# usage: bash tools/sweep_cfg.sh <tag> <config> "<args1>" "<args2>" ...
tag=$1; cfg=$2; shift; shift
for a in "$@"; do
  timeout 600 python bench.py --config $cfg --steps 20 --warmup 3 --no-cpu-baseline --e2e-steps 1 $a > gpurun_out/sweep_${tag}.tmp 2>&1
  echo "== $cfg $a" >> gpurun_out/sweep_${tag}.log
  tail -1 gpurun_out/sweep_${tag}.tmp >> gpurun_out/sweep_${tag}.log
done
rm -f gpurun_out/sweep_${tag}.tmp
