# paired scatter: parity, then c3 / c4 phases with scatter_pair 1 (default) vs 0
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_bucketed.py tests/test_gpu_fuzz.py tests/test_gpu_sharded.py tests/test_gpu_placement.py -m gpu -x -q -p no:cacheprovider > gpurun_out/s5d_pytest.log 2>&1; echo rc=$? >> gpurun_out/s5d_pytest.log
bash tools/sweep_cfg.sh s5d c3 "" "--param scatter_pair=0" "" "--param scatter_pair=0"
bash tools/sweep_cfg.sh s5d c4 "" "--param scatter_pair=0"
