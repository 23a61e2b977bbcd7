#!/bin/bash
# C5 probe variants, a launch-time list of one run, then one ncu --set full capture of chosen kernels
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
timeout 900 python scripts/probe_c5.py 512 "" ${PROBE_VARIANTS} > gpurun_out/probe.jsonl 2> gpurun_out/probe.err
echo "probe rc=$?" >> gpurun_out/probe.err
if [ -z "$NO_LIST" ]; then
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv \
  --log-file gpurun_out/launches.csv python scripts/probe_c5.py 512 > gpurun_out/ncu_list.log 2>&1
echo "ncu list rc=$?" >> gpurun_out/ncu_list.log
fi
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"${NCU_K:-k_grs_emit|k_grs_walk}" -c ${NCU_C:-2} --launch-skip ${NCU_SKIP:-2} \
  -o gpurun_out/grs -f python scripts/probe_c5.py 512 > gpurun_out/ncu.log 2>&1
echo "ncu rc=$?" >> gpurun_out/ncu.log
