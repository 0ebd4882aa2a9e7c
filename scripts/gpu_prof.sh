#!/bin/bash
# Build, event counters (blastp_debug_stats on configs 1-3), one ncu --set full capture
# of the config-3 search kernel (+ a short bench).  PROF names the .ncu-rep.
mkdir -p gpurun_out
python -c "from paper_conf_ipps_zhangwlf14_b200 import build; build.build()" > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
timeout 600 python scripts/stats.py gpurun_out/stats.json > gpurun_out/stats.txt 2>&1; echo "stats rc=$?"; cat gpurun_out/stats.txt | tail -40
timeout 600 python bench.py --steps 20 --warmup 3 --no-cpu-baseline --no-e2e ${BENCH_ARGS:-} > gpurun_out/bench_quick.json 2> gpurun_out/bench_quick.err; echo "bench rc=$?"
python -c "
import json;d=json.load(open('gpurun_out/bench_quick.json'));print('value',d['value'],'ms',d['ms_per_step'],'clk',d['clocks'])"
K=${KREGEX:-search_}
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:$K -s 1 -c 1 \
  -o gpurun_out/${PROF:-prof} -f python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline ${BENCH_ARGS:-} > gpurun_out/ncu_full.log 2>&1
echo "ncu rc=$?"
