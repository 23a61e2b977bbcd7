#!/bin/bash
# quick GPU check: GRS-affected tests, then per-kernel C5 timings (scripts/probe_c5.py)
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_validate.py tests/test_gpu_c5.py ${PYTEST_EXTRA} -x -q ${PYTEST_K:+-k "$PYTEST_K"} > gpurun_out/pytest_quick.txt 2>&1
echo "rc=$?" >> gpurun_out/pytest_quick.txt
timeout 600 python scripts/probe_c5.py 512 "" ${PROBE_VARIANTS} > gpurun_out/probe.jsonl 2> gpurun_out/probe.err
echo "probe rc=$?" >> gpurun_out/probe.err
