#!/bin/bash
# round-2 GPU session: tests + C5 bench (outputs under gpurun_out/)
cd "$GRAFT_REPO_ROOT" || exit 1
nvidia-smi --query-gpu=name,memory.total,clocks.sm --format=csv > gpurun_out/smi.txt 2>&1
free -g > gpurun_out/free.txt
timeout 1500 python -m pytest tests -m gpu -x -q ${PYTEST_K:+-k "$PYTEST_K"} > gpurun_out/pytest_gpu.txt 2>&1
echo "pytest rc=$?" >> gpurun_out/pytest_gpu.txt
timeout 900 python bench.py ${BENCH_ARGS} > gpurun_out/bench.json 2> gpurun_out/bench.err
echo "bench rc=$?" >> gpurun_out/bench.err
