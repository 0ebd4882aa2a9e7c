#!/bin/bash
# Round-end evidence: build; ncu --set full of the config-3 search kernel (one launch) ->
# profiles json via capture_json.py (tagged with the csrc hash); the launch list of a short
# bench (gpu__time_duration.sum); per-region instruction breakdown inputs.
mkdir -p gpurun_out
python -c "from paper_conf_ipps_zhangwlf14_b200 import build; build.build()" > gpurun_out/build.log 2>&1 || exit 1
cp paper_conf_ipps_zhangwlf14_b200/build/search_block.cu.o gpurun_out/search_block_final.cu.o
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:search_block_kernel -s 1 -c 1 \
  -o gpurun_out/prof_final -f python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/ncu_full.log 2>&1
echo "ncu full rc=$?"
timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file gpurun_out/launches_final.csv python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/ncu_launches.log 2>&1
echo "ncu launches rc=$?"
