cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_bucketed.py -x -q > gpurun_out/r02d_bucketed.log 2>&1; echo "rc=$?" >> gpurun_out/r02d_bucketed.log
timeout 900 python tools/param_sweep.py --config c4 --steps 10 --set item_dir32=0 --set item_dir32=1 --set item_dir32=0 --set item_dir32=1 > gpurun_out/r02d_c4_dir32.jsonl 2>&1
timeout 600 python tools/param_sweep.py --config c5 --steps 20 --set item_dir32=0 --set item_dir32=1 --set item_dir32=0 --set item_dir32=1 > gpurun_out/r02d_c5_dir32.jsonl 2>&1
timeout 1200 python -m pytest tests/test_gpu_c4_full.py -x -q > gpurun_out/r02d_c4full.log 2>&1; echo "rc=$?" >> gpurun_out/r02d_c4full.log
