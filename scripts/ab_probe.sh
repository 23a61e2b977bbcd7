#!/bin/bash
# A/B of compile-time variants on the C5 probe: bash scripts/ab_probe.sh "name:flags" ...
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out /tmp/lfab
for spec in "$@"; do
  name=${spec%%:*}; flags=${spec#*:}
  python scripts/build_variant.py /tmp/lfab/$name.so $flags > gpurun_out/ab_$name.build 2>&1 || { echo "$name build failed"; continue; }
done
for spec in "$@"; do
  name=${spec%%:*}
  [ -f /tmp/lfab/$name.so ] || continue
  LF_LIB_PATH=/tmp/lfab/$name.so timeout 600 python scripts/probe_c5.py ${AB_N:-512} ${AB_ENV:-""} > gpurun_out/ab_$name.jsonl 2> gpurun_out/ab_$name.err
done
