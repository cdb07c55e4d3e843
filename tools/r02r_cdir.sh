cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
TAG=${1:-r02r}
timeout 1800 python -m pytest tests/test_gpu_bucketed.py tests/test_gpu_regular.py tests/test_gpu_c4_full.py tests/test_gpu_sharded.py tests/test_gpu_concurrency.py -x -q > gpurun_out/${TAG}_tests.log 2>&1; echo "rc=$?" >> gpurun_out/${TAG}_tests.log
for c in c3 c5; do timeout 900 python tools/param_sweep.py --config $c --steps 20 --set item_cdir=1 --set item_cdir=0 --set item_cdir=1 --set item_cdir=0 > gpurun_out/${TAG}_$c.jsonl 2>&1; done
timeout 900 python tools/param_sweep.py --config c4 --steps 10 --set item_cdir=1 --set item_cdir=0 --set item_cdir=1 > gpurun_out/${TAG}_c4.jsonl 2>&1
