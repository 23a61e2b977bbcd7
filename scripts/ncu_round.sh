#!/bin/bash
# launch list + full captures of selected kernels; usage: ncu_round.sh tag "regex" count
TAG=$1; RE=${2:-"k_propose_tile|k_lf_local1|k_red_scan|k_rounds_fused"}; C=${3:-6}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
  --log-file gpurun_out/launches_$TAG.csv python bench.py --steps 2 --warmup 1 --no-graph --no-cpu-baseline \
  > gpurun_out/ncu_launch_$TAG.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"$RE" -c $C \
  -o gpurun_out/prof_$TAG -f python bench.py --steps 1 --warmup 1 --no-graph --no-cpu-baseline \
  > gpurun_out/ncu_full_$TAG.log 2>&1
echo done
