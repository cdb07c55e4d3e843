# all 1-GPU configs, one JSON line each into gpurun_out/configs.log
timeout 900 python -m pytest tests/test_gpu_implicit.py -x -q > gpurun_out/pytest_impl.log 2>&1
tail -1 gpurun_out/pytest_impl.log
for c in c2 c1 c3 c5 c4; do
  extra="--no-cpu-baseline"
  [ "$c" = "c2" ] && extra=""
  echo "== $c" >> gpurun_out/configs.log
  timeout 900 python bench.py --config $c --steps 100 --warmup 5 $extra > gpurun_out/bench_$c.log 2>&1
  tail -1 gpurun_out/bench_$c.log >> gpurun_out/configs.log
done
