#!/bin/bash
# Full measurement session under gpurun: build, GPU tests, smoke, bench, ncu launch list,
# ncu --set full of the step's kernels, phase-timing variant.  usage: gpu_session.sh TAG [what...]
set -u
TAG=$1; shift
WHAT=${*:-"tests smoke bench ncu phase"}
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total --format=csv > gpurun_out/gpu_$TAG.txt 2>&1
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_$TAG.log 2>&1 || echo BUILD FAILED
for w in $WHAT; do
  case $w in
    tests)
      timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu_$TAG.log 2>&1
      echo "pytest rc=$?" >> gpurun_out/pytest_gpu_$TAG.log ;;
    quick)
      timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "small or edge or long or full_c2 or native" > gpurun_out/pytest_gpu_$TAG.log 2>&1
      echo "pytest rc=$?" >> gpurun_out/pytest_gpu_$TAG.log ;;
    smoke)
      timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_$TAG.log 2>&1
      echo "smoke rc=$?" >> gpurun_out/smoke_$TAG.log ;;
    bench)
      timeout 600 python bench.py --steps 20 --warmup 5 > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err ;;
    benchfast)
      timeout 600 python bench.py --steps 20 --warmup 5 --no-cpu-baseline > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err ;;
    ncu)
      timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
        --log-file gpurun_out/launches_$TAG.csv python bench.py --steps 2 --warmup 1 --no-graph --no-cpu-baseline \
        > gpurun_out/ncu_launch_$TAG.log 2>&1
      timeout 900 ncu --set full --clock-control none --import-source on \
        -k regex:"k_propose_stream|k_mutual0|k_rounds_fused|k_lf_full1|k_red_full|k_lf_full2|k_perm_tri" -c 7 \
        -o gpurun_out/prof_$TAG -f python bench.py --steps 1 --warmup 1 --no-graph --no-cpu-baseline \
        > gpurun_out/ncu_full_$TAG.log 2>&1 ;;
    phase)
      bash scripts/variants.sh ${TAG} "phase:-DLF_PHASE_TIMING" > gpurun_out/var_$TAG.log 2>&1 ;;
  esac
done
echo done
