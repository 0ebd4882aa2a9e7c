#!/bin/bash
# Instructions / duration / issue metrics of the search kernel for several library builds
# (one short ncu pass each, config 3 unless BENCH_ARGS says otherwise).
mkdir -p gpurun_out
for lib in "$@"; do
  echo "== $(basename "$lib")"
  BLASTP_LIB=$(realpath "$lib") timeout 900 ncu --clock-control none -k regex:search_ -s 1 -c 1 \
    --metrics gpu__time_duration.sum,smsp__inst_executed.sum,smsp__thread_inst_executed_per_inst_executed.ratio,sm__warps_active.avg.pct_of_peak_sustained_active,smsp__issue_active.avg.pct_of_peak_sustained_active \
    python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline ${BENCH_ARGS:-} 2>&1 | grep -E "search_|duration|inst_executed|warps_active|issue_active" | head -8
done
