cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
timeout 600 python scripts/probe_c5.py C3 "" "LF_ROWS_SPLIT=1" "LF_FOREST=grs,LF_GRS_SHIFT=28" "LF_ROWS_SPLIT=1,LF_FOREST=grs,LF_GRS_SHIFT=28" > gpurun_out/probe_c3.jsonl 2> gpurun_out/probe_c3.err
timeout 600 python scripts/probe_c5.py C4 "" "LF_GRS_SHIFT=28" > gpurun_out/probe_c4.jsonl 2>> gpurun_out/probe_c3.err
