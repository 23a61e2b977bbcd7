#!/bin/bash
# quick check: the C5 test file (with memcheck on failure), then all GPU tests, then bench
cd "$GRAFT_REPO_ROOT" || exit 1
timeout 900 python -m pytest tests/test_gpu_c5.py -x -q -k "64" > gpurun_out/pytest_c5small.txt 2>&1
rc=$?
echo "rc=$rc" >> gpurun_out/pytest_c5small.txt
if [ $rc -ne 0 ]; then
  timeout 600 compute-sanitizer --tool memcheck --print-limit 20 python -m pytest tests/test_gpu_c5.py -x -q -k "64_digests" > gpurun_out/memcheck_c5small.txt 2>&1
  exit 1
fi
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.txt 2>&1
echo "pytest rc=$?" >> gpurun_out/pytest_gpu.txt
timeout 900 python bench.py ${BENCH_ARGS} > gpurun_out/bench.json 2> gpurun_out/bench.err
echo "bench rc=$?" >> gpurun_out/bench.err
