#!/bin/bash
# C5: ncu launch list of bench steps (time, DRAM bytes, warp instructions) + one --set full
# capture of the chosen kernels (second step); outputs in gpurun_out/
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,smsp__inst_executed.sum \
  --clock-control none --csv --log-file gpurun_out/launches_c5.csv \
  python bench.py --steps 2 --warmup 1 --no-graph --no-cpu-baseline --no-e2e --extra "" > gpurun_out/ncu_list.log 2>&1
echo "list rc=$?" >> gpurun_out/ncu_list.log
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:"${NCU_K:-k_rows_propose_k|k_grs_walk|k_grs_emit|k_propose_stream}" \
  -c ${NCU_C:-7} --launch-skip ${NCU_SKIP:-0} -o gpurun_out/c5_full -f \
  python bench.py --steps 1 --warmup 1 --no-graph --no-cpu-baseline --no-e2e --extra "" > gpurun_out/ncu_full.log 2>&1
echo "full rc=$?" >> gpurun_out/ncu_full.log
