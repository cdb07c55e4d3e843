set -x
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; tail -3 gpurun_out/pytest_gpu.log
for cfg in "--qpl 1 --threads 512" "--qpl 2 --threads 512" "--qpl 1 --threads 256" "--qpl 2 --threads 256" "--qpl 1 --smem 200000" "--qpl 2 --smem 200000"; do
  timeout 300 python bench.py --steps 200 --warmup 5 --no-cpu-baseline --e2e-steps 1 $cfg 2>&1 | python -c "import json,sys; d=json.loads(sys.stdin.readlines()[-1]); print('$cfg', d['value'], d['ms_per_step'], d['roofline_l2']['frac'], d['roofline']['frac'])"
done
