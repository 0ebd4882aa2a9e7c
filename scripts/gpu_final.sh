#!/bin/bash
# Round-end evidence on one GPU: the whole GPU test suite, then
# scripts/gpu_measure.sh (launch list, ncu capture + summary, bench line, sweep).
# Usage: bash scripts/gpu_final.sh <label> [round]
mkdir -p gpurun_out
timeout 1800 python -m pytest tests -m gpu -q --durations=10 > gpurun_out/pytest_gpu.log 2>&1
tail -14 gpurun_out/pytest_gpu.log
bash scripts/gpu_measure.sh "$@"
