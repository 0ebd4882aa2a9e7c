#!/bin/bash
# Parity subset of a candidate library build (BLASTP_LIB), then an interleaved
# A/B of library builds on config 3.  Usage: bash scripts/gpu_ab_parity.sh <cand.so> <rounds> <lib>...
mkdir -p gpurun_out
cand=$1; rounds=$2; shift 2
BLASTP_LIB=$(realpath "$cand") timeout 900 python -m pytest tests -m gpu -q -x -k "(test_gpu_parity and warp and (config1 or config2 or fuzz or adversarial or long_subjects or edge or long_query or config3 or stats)) or (stateful and warp)" > gpurun_out/pytest_cand.log 2>&1
tail -3 gpurun_out/pytest_cand.log
bash scripts/ab.sh "$rounds" "$@" 2>&1 | tee gpurun_out/ab.txt
