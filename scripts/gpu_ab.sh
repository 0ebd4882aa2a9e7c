#!/bin/bash
# Parity subset on the in-tree library, then an interleaved A/B of library
# builds on config 3 (device time), then kernel event counters.
# Usage (GPU box): bash scripts/gpu_ab.sh <rounds> <lib1.so> <lib2.so> ...
mkdir -p gpurun_out
rounds=$1; shift
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "warp and (config1 or fuzz or adversarial or long_subjects or config3 or edge or long_query)" > gpurun_out/pytest_ab.log 2>&1
tail -3 gpurun_out/pytest_ab.log
bash scripts/ab.sh "$rounds" "$@" 2>&1 | tee gpurun_out/ab.txt
timeout 300 python scripts/stats.py gpurun_out/stats.json > gpurun_out/stats.txt 2>&1; tail -30 gpurun_out/stats.txt
