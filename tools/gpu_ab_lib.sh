#!/bin/bash
# A/B of two in-tree builds (libhbt_base.so vs libhbt.so), alternating: tools/gpu_ab_lib.sh CONFIG TAG [steps]
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
C=$1; TAG=$2; S=${3:-10}
for i in 1 2 3; do
  HBT_LIB_ALT=libhbt_base.so timeout 600 python tools/param_sweep.py --config $C --steps $S | sed 's/^{/{"lib": "base", /' >> gpurun_out/${TAG}.jsonl 2>&1
  timeout 600 python tools/param_sweep.py --config $C --steps $S | sed 's/^{/{"lib": "new", /' >> gpurun_out/${TAG}.jsonl 2>&1
done
