#!/bin/bash
# round-2 GPU session 1: new full-size parity tests, default bench (c4), 2-rank dry run, reference arm
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,memory.total --format=csv > gpurun_out/r02g1_smi.txt
timeout 1500 python -m pytest tests/test_gpu_c4_full.py "tests/test_gpu_bucketed.py::test_c3_full_size_bench_launch" -x -q > gpurun_out/r02g1_fulltests.log 2>&1
echo "fulltests rc=$?" >> gpurun_out/r02g1_fulltests.log
timeout 900 python bench.py --steps 20 --warmup 5 > gpurun_out/r02g1_bench.jsonl 2> gpurun_out/r02g1_bench.err
echo "bench rc=$?" >> gpurun_out/r02g1_bench.err
timeout 900 python bench.py --gpus 2 --steps 10 --warmup 3 > gpurun_out/r02g1_bench_g2.jsonl 2> gpurun_out/r02g1_bench_g2.err
echo "bench g2 rc=$?" >> gpurun_out/r02g1_bench_g2.err
timeout 600 python bench.py --impl reference --steps 5 --warmup 1 > gpurun_out/r02g1_ref.jsonl 2> gpurun_out/r02g1_ref.err
