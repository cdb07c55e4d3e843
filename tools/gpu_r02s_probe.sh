cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 300 python tools/gather_probe.py > gpurun_out/r02s_gather_probe.jsonl 2>&1
timeout 900 python tools/param_sweep.py --config c4 --steps 10 --set item_qprefetch=0 --set item_qprefetch=1 --set item_qprefetch=0 --set item_qprefetch=1 > gpurun_out/r02s_c4_qprefetch_ab.jsonl 2>&1
