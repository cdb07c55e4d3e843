cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
TAG=${1:-r02n}
timeout 1200 python -m pytest tests/test_gpu_bucketed.py tests/test_gpu_c4_full.py tests/test_gpu_sharded.py -x -q > gpurun_out/${TAG}_tests.log 2>&1; echo "rc=$?" >> gpurun_out/${TAG}_tests.log
python tools/c4_ties_check.py 26 24 20000000 > gpurun_out/${TAG}_ties.log 2>&1
timeout 900 python tools/param_sweep.py --config c4 --steps 10 --set item_dir32=1 --set item_dir32=0 --set item_dir32=1 > gpurun_out/${TAG}_c4.jsonl 2>&1
timeout 600 python tools/param_sweep.py --config c5 --steps 20 --set item_dir32=1 --set item_dir32=0 --set item_dir32=1 > gpurun_out/${TAG}_c5.jsonl 2>&1
