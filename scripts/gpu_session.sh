#!/bin/bash
# One GPU session: tests, bench, launch list, ncu capture of the search kernel.
# Usage (on the GPU box via gpurun): bash scripts/gpu_session.sh [tests|bench|ncu|all]
set -u
mkdir -p gpurun_out
what=${1:-all}
if [[ $what == tests || $what == all ]]; then
  timeout 1500 python -m pytest tests -m gpu -q --durations=15 > gpurun_out/pytest_gpu.log 2>&1
  tail -25 gpurun_out/pytest_gpu.log
fi
if [[ $what == bench || $what == all ]]; then
  timeout 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err
  echo "bench rc=$?"; tail -3 gpurun_out/bench.err; cat gpurun_out/bench.json
fi
if [[ $what == ncu || $what == all ]]; then
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
    --log-file gpurun_out/launches.csv python bench.py --steps 3 --warmup 3 --no-e2e \
    --no-cpu-baseline > gpurun_out/ncu_launch_bench.json 2>&1
  echo "ncu launches rc=$?"
  timeout 1200 ncu --set full --clock-control none --import-source on -k regex:search_ \
    -s 3 -c 1 -o gpurun_out/prof_search python bench.py --steps 2 --warmup 3 --no-e2e \
    --no-cpu-baseline > gpurun_out/ncu_full.log 2>&1
  echo "ncu full rc=$?"; tail -3 gpurun_out/ncu_full.log
fi
