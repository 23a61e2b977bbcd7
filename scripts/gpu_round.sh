#!/bin/bash
# One gpurun session: build, GPU tests, smoke, bench, ncu launch list + full capture.
# usage (from the repo root, under gpurun): bash scripts/gpu_round.sh [tag] [what...]
set -u
TAG=${1:-r01}
shift || true
WHAT=${*:-"tests smoke bench ncu"}
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total --format=csv > gpurun_out/gpu_$TAG.txt 2>&1
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_$TAG.log 2>&1 || echo BUILD FAILED
for w in $WHAT; do
  case $w in
    tests)
      timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu_$TAG.log 2>&1
      echo "pytest rc=$?" >> gpurun_out/pytest_gpu_$TAG.log ;;
    quicktests)
      timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "small or edge or long or schedules or maximal or native" > gpurun_out/pytest_gpu_$TAG.log 2>&1
      echo "pytest rc=$?" >> gpurun_out/pytest_gpu_$TAG.log ;;
    smoke)
      timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_$TAG.log 2>&1
      echo "smoke rc=$?" >> gpurun_out/smoke_$TAG.log ;;
    bench)
      timeout 600 python bench.py --steps 20 --warmup 5 > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err ;;
    ncu)
      timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 200 --csv \
        --log-file gpurun_out/launches_$TAG.csv python bench.py --steps 2 --warmup 1 --no-graph --no-cpu-baseline \
        > gpurun_out/ncu_bench_$TAG.log 2>&1
      timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_propose -c 2 \
        -o gpurun_out/prof_propose_$TAG -f python bench.py --steps 1 --warmup 1 --no-graph --no-cpu-baseline \
        > gpurun_out/ncu_full_propose_$TAG.log 2>&1
      timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_cycle_scan|k_rank_scan|k_mutual" -c 4 \
        -o gpurun_out/prof_lf_$TAG -f python bench.py --steps 1 --warmup 1 --no-graph --no-cpu-baseline \
        > gpurun_out/ncu_full_lf_$TAG.log 2>&1 ;;
  esac
done
echo done
