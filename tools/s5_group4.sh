# 4-lane groups in the implicit item search: parity, then c4 A/B
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_bucketed.py tests/test_gpu_fuzz.py -m gpu -x -q -p no:cacheprovider > gpurun_out/s5e_pytest.log 2>&1; echo rc=$? >> gpurun_out/s5e_pytest.log
bash tools/sweep_cfg.sh s5e c4 "" "--param item_group4=1" "" "--param item_group4=1"
bash tools/sweep_cfg.sh s5e c5 "--bucket 1" "--bucket 1 --param item_group4=1"
