#!/bin/bash
# generic GPU session: TESTS (pytest args, optional) then BENCH_ARGS (optional) -> gpurun_out/
cd "$GRAFT_REPO_ROOT" || exit 1
if [ -n "$TESTS" ]; then
  timeout ${TEST_TIMEOUT:-1500} python -m pytest $TESTS -x -q > gpurun_out/pytest.txt 2>&1
  rc=$?
  echo "pytest rc=$rc" >> gpurun_out/pytest.txt
  if [ $rc -ne 0 ] && [ -n "$MEMCHECK" ]; then
    timeout 900 compute-sanitizer --tool memcheck --print-limit 10 python -m pytest $MEMCHECK -x -q > gpurun_out/memcheck.txt 2>&1
  fi
  [ $rc -ne 0 ] && [ -z "$BENCH_ANYWAY" ] && exit 1
fi
if [ -n "$BENCH_ARGS" ]; then
  timeout ${BENCH_TIMEOUT:-900} python bench.py $BENCH_ARGS > gpurun_out/bench.json 2> gpurun_out/bench.err
  echo "bench rc=$?" >> gpurun_out/bench.err
fi
if [ -n "$EXTRA" ]; then
  bash -c "$EXTRA" > gpurun_out/extra.txt 2>&1
fi
