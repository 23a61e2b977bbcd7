cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out /tmp/lfab
for spec in "$@"; do
  name=${spec%%:*}; flags=${spec#*:}
  python scripts/build_variant.py /tmp/lfab/$name.so $flags > /dev/null 2>&1
  LF_LIB_PATH=/tmp/lfab/$name.so timeout 300 python scripts/probe_c5.py C2 "" | sed "s/^/$name /" >> gpurun_out/ab_c2.txt 2>&1
done
