cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 1500 python -m pytest tests -x -q -m gpu > gpurun_out/r02s_pytest_gpu.log 2>&1; echo "rc=$?" >> gpurun_out/r02s_pytest_gpu.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r02s_smoke.log 2>&1
timeout 900 python bench.py > gpurun_out/r02s_bench_default.log 2>&1
