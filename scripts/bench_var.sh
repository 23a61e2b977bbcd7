cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
timeout 600 python bench.py --steps 10 --warmup 3 --extra "" --no-e2e --no-cpu-baseline > gpurun_out/b_graph.json 2>/dev/null
LF_NO_PDL=1 timeout 600 python bench.py --steps 10 --warmup 3 --extra "" --no-e2e --no-cpu-baseline > gpurun_out/b_nopdl.json 2>/dev/null
timeout 600 python bench.py --steps 10 --warmup 3 --extra "" --no-e2e --no-cpu-baseline --no-graph > gpurun_out/b_eager.json 2>/dev/null
