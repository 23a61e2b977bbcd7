cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
timeout 600 python scripts/probe_c5.py C4 "" "LF_WALK_BPSM=2" "LF_WALK_BPSM=4" > gpurun_out/probe_c4.jsonl 2> gpurun_out/probe_c4.err
timeout 600 python scripts/probe_c5.py 512 "" > gpurun_out/probe.jsonl 2> gpurun_out/probe.err
