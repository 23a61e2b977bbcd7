cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
for c in C2 C3 C4; do
  timeout 600 python scripts/probe_c5.py $c "LF_FOREST=tile" "LF_FOREST=grs" "LF_FOREST=grs,LF_GRS_SHIFT=26" "LF_FOREST=grs,LF_GRS_SHIFT=28" >> gpurun_out/probe_cfg.jsonl 2>> gpurun_out/probe_cfg.err
done
