#!/bin/bash
# Build compile-time variants of liblf.so and bench each (kernel breakdown + headline).
# usage (repo root, under gpurun): bash scripts/variants.sh tag "name:flags" ["name:flags" ...]
#   e.g. bash scripts/variants.sh r01t "base:" "lt1024:-DLF_LT=1024"
# A variant named *phase* is also run through the forest-stats phase dump.
set -u
TAG=$1; shift
mkdir -p gpurun_out /tmp/lfvar
for spec in "$@"; do
  name=${spec%%:*}; flags=${spec#*:}
  LF_EXTRA_FLAGS="$flags" python -c "from paper_conf_icpp_0002s22_b200 import _build as b; b.build(force=True)" \
    > gpurun_out/var_${TAG}_${name}.build 2>&1 || { echo "$name BUILD FAILED"; continue; }
  cp paper_conf_icpp_0002s22_b200/liblf.so /tmp/lfvar/$name.so
done
for spec in "$@"; do
  name=${spec%%:*}
  [ -f /tmp/lfvar/$name.so ] || continue
  if [[ $name == *quick* ]]; then
    LF_LIB_PATH=/tmp/lfvar/$name.so timeout 900 python -m pytest tests/test_gpu_parity.py -x -q \
      -k "small or edge or long or full_c2" > gpurun_out/var_${TAG}_${name}.pytest 2>&1
    echo "pytest rc=$?" >> gpurun_out/var_${TAG}_${name}.pytest
  fi
  LF_LIB_PATH=/tmp/lfvar/$name.so timeout 300 python bench.py --steps 20 --warmup 5 --no-cpu-baseline \
    > gpurun_out/var_${TAG}_${name}.json 2> gpurun_out/var_${TAG}_${name}.err
  echo "$name rc=$?"
done
# restore the default build
python -c "from paper_conf_icpp_0002s22_b200 import _build as b; b.build(force=True)" > /dev/null 2>&1
echo done
