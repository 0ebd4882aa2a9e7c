#!/bin/bash
# Tests named by a pytest -k expression (or all GPU tests), then an interleaved
# A/B of library builds on config 3.  Usage: bash scripts/gpu_check.sh "<k-expr>" <rounds> <lib>...
mkdir -p gpurun_out
k=$1; rounds=$2; shift 2
if [[ -n $k ]]; then
  timeout 1500 python -m pytest tests -m gpu -q -x -k "$k" --durations=10 > gpurun_out/pytest_check.log 2>&1
else
  timeout 1500 python -m pytest tests -m gpu -q --durations=10 > gpurun_out/pytest_check.log 2>&1
fi
tail -15 gpurun_out/pytest_check.log
if [[ $rounds -gt 0 ]]; then bash scripts/ab.sh "$rounds" "$@" 2>&1 | tee gpurun_out/ab.txt; fi
