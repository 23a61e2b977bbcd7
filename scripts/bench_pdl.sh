cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
for c in C2 C3 C4; do
  timeout 600 python bench.py --config $c --steps 20 --warmup 5 --extra "" --no-e2e --no-cpu-baseline > gpurun_out/p_$c.json 2>/dev/null
  LF_NO_PDL=1 timeout 600 python bench.py --config $c --steps 20 --warmup 5 --extra "" --no-e2e --no-cpu-baseline > gpurun_out/p_${c}_nopdl.json 2>/dev/null
done
