#!/bin/bash
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 1200 python tools/e2e_sweep.py > gpurun_out/r02g14_e2e.jsonl 2> gpurun_out/r02g14_e2e.err
