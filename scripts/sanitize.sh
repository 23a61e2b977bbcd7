#!/bin/bash
# compute-sanitizer memcheck / racecheck / synccheck / initcheck over scripts/sanitize_cases.py
cd "$GRAFT_REPO_ROOT" || exit 1
for tool in memcheck racecheck synccheck initcheck; do
  extra=""
  [ "$tool" = "racecheck" ] && extra="--racecheck-report analysis"
  timeout 1500 compute-sanitizer --tool $tool $extra --print-limit 200 python scripts/sanitize_cases.py \
    > gpurun_out/sanitizer_$tool.txt 2>&1
  echo "rc=$?" >> gpurun_out/sanitizer_$tool.txt
done
