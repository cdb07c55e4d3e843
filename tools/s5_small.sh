# small-batch CTA size: parity (fuzz), then c1 A/B
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_fuzz.py tests/test_gpu_implicit.py -m gpu -x -q -p no:cacheprovider > gpurun_out/s5g_pytest.log 2>&1; echo rc=$? >> gpurun_out/s5g_pytest.log
bash tools/sweep_cfg.sh s5g c1 "" "--param small_threads=128" "" "--param small_threads=128" "--param small_threads=1024"
