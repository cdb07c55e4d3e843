# L2 hint A/B, round 2: parity under the hints, c3 item search, c5 uniform, c2 / c1 repeats
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_bucketed.py tests/test_gpu_fuzz.py -m gpu -x -q -p no:cacheprovider > gpurun_out/hint_pytest.log 2>&1; echo rc=$? >> gpurun_out/hint_pytest.log
bash tools/sweep_cfg.sh hint2 c3 "" "--param item_l2_hint=1" "--param item_l2_hint=2" "--param item_l2_hint=3"
bash tools/sweep_cfg.sh hint2 c5 "--queries uniform_values" "--queries uniform_values --param l2_hint=1"
bash tools/sweep_cfg.sh hint2 c2 "" "--param l2_hint=1" "" "--param l2_hint=1"
bash tools/sweep_cfg.sh hint2 c1 "" "--param l2_hint=1"
