cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out /tmp/lfab
python scripts/build_variant.py /tmp/lfab/base.so > /dev/null 2>&1
python scripts/build_variant.py /tmp/lfab/s128.so -DLF_SPT=128 -DLF_SETILE_BIG=4096 > /dev/null 2>&1
python scripts/build_variant.py /tmp/lfab/s64.so -DLF_SPT=64 -DLF_SETILE_BIG=2048 > /dev/null 2>&1
for v in base s128 s64; do for c in C2 C3 C4 512; do
  LF_LIB_PATH=/tmp/lfab/$v.so timeout 300 python scripts/probe_c5.py $c "" | sed "s/^/$v /" >> gpurun_out/ab_multi.txt 2>&1
done; done
