#!/bin/bash
# ncu --set full on selected kernels of one bench step (no graph); usage: prof_kernels.sh tag regex count
TAG=$1; RE=$2; C=${3:-4}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"$RE" -c $C \
  -o gpurun_out/prof_$TAG -f python bench.py --steps 1 --warmup 1 --no-graph --no-cpu-baseline \
  > gpurun_out/ncu_$TAG.log 2>&1
echo rc=$?
