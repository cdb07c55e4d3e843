for a in "" "--param host_chunk_log2=20" "--param host_chunk_log2=21" "--param host_bufs=3" "--param host_chunk_log2=20 --param host_bufs=3" "--param host_chunk_log2=21 --param host_bufs=3" "--param host_chunk_log2=20 --param host_bufs=4"; do
  timeout 600 python bench.py --config c2 --steps 20 --warmup 3 --no-cpu-baseline --e2e-steps 10 $a > gpurun_out/e2e.tmp 2>&1
  echo "== $a" >> gpurun_out/sweep_e2e.log; tail -1 gpurun_out/e2e.tmp >> gpurun_out/sweep_e2e.log
done
