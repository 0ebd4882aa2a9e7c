#!/bin/bash
# A/B device timing of library builds on one box, interleaved to cancel drift.
# Usage: bash scripts/ab.sh <rounds> <lib1.so> <lib2.so> ... (BENCH_ARGS passed to bench.py)
mkdir -p gpurun_out
rounds=$1; shift
for r in $(seq "$rounds"); do
  for lib in "$@"; do
    v=$(BLASTP_LIB=$(realpath "$lib") timeout 600 python bench.py --steps 10 --warmup 3 --no-e2e \
        --no-cpu-baseline ${BENCH_ARGS:-} 2>/dev/null |
        python -c "import json,sys; d=json.loads(sys.stdin.read()); print(f\"{d['ms_per_step']:.3f}\")")
    echo "round $r  $(basename "$lib")  ms/step $v"
  done
done
