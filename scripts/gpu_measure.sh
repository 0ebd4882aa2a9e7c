#!/bin/bash
# Measurement session (one GPU): ncu launch list + one full capture of the
# search kernel, summarised into profiles/<round>/ (bench.py reads the
# instruction count and DRAM bytes from profiles/ncu_search_kernel.json), then
# the bench line and the strategy sweep.  Results copied to gpurun_out/.
# Usage: bash scripts/gpu_measure.sh <label> [round]
set -u
label=$1; rnd=${2:-r01}
mkdir -p gpurun_out
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file gpurun_out/launches.csv python bench.py --steps 3 --warmup 3 --no-e2e \
  --no-cpu-baseline > gpurun_out/ncu_launch_bench.json 2>&1
echo "ncu launches rc=$?"
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:search_ \
  -s 3 -c 1 -o gpurun_out/prof_search python bench.py --steps 2 --warmup 3 --no-e2e \
  --no-cpu-baseline > gpurun_out/ncu_full.log 2>&1
echo "ncu full rc=$?"
python scripts/summarize_ncu.py gpurun_out/prof_search.ncu-rep gpurun_out/launches.csv \
  profiles/$rnd $label > gpurun_out/summary.txt 2>&1; echo "summary rc=$?"
mkdir -p gpurun_out/profiles/$rnd
cp profiles/$rnd/*$label* gpurun_out/profiles/$rnd/ 2>/dev/null
cp profiles/ncu_search_kernel.json gpurun_out/profiles/
timeout 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?"
cat gpurun_out/bench.json
timeout 1200 python scripts/sweep.py gpurun_out/sweep.json 5 > gpurun_out/sweep.txt 2>&1; echo "sweep rc=$?"
tail -40 gpurun_out/sweep.txt
