#!/bin/bash
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 2400 python -m pytest tests -x -q -m gpu > gpurun_out/r02g11_gpu.log 2>&1
echo "rc=$?" >> gpurun_out/r02g11_gpu.log
bash tools/sanitize.sh
timeout 900 python bench.py --steps 20 --warmup 5 > gpurun_out/r02g11_bench.jsonl 2> gpurun_out/r02g11_bench.err
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r02g11_smoke.log 2>&1
