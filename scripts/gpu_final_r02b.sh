#!/bin/bash
# Round-2 final evidence (second session): the default bench line, one ncu
# --set full capture of the config-3 search kernel (-> profiles/ncu_search_kernel.json,
# tagged with the csrc hash), the launch list of a short bench, full captures of the
# gapped stage's two DP kernels, the Fig. 12 overlap re-measured.
mkdir -p gpurun_out
python -c "from paper_conf_ipps_zhangwlf14_b200 import build; build.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 900 python bench.py > gpurun_out/bench_final.json 2> gpurun_out/bench_final.err; echo "bench rc=$?"
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:search_block_kernel -s 1 -c 1 \
  -o gpurun_out/prof_final -f python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --no-gapped > gpurun_out/ncu_full.log 2>&1
echo "ncu search rc=$?"
timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file gpurun_out/launches_final.csv python bench.py --steps 3 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/ncu_launches.log 2>&1
echo "ncu launches rc=$?"
python scripts/summarize_ncu.py gpurun_out/prof_final.ncu-rep gpurun_out/launches_final.csv gpurun_out/profiles/r02 search_kernel_r02b > gpurun_out/summary.txt 2>&1; echo "summary rc=$?"
python scripts/capture_json.py gpurun_out/prof_final.ncu-rep gpurun_out/ncu_search_kernel.json > /dev/null 2>&1; echo "capture_json rc=$?"
PYTHONPATH=. timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"gapped_(warp|trace)" \
  -c 2 -o gpurun_out/prof_gapped_final -f python scripts/gapped_time.py > gpurun_out/ncu_gapped.log 2>&1; echo "ncu gapped rc=$?"
PYTHONPATH=. timeout 900 python scripts/gapped_pipe_time.py > gpurun_out/gapped_pipe.txt 2>&1; echo "pipe rc=$?"; cat gpurun_out/gapped_pipe.txt
python -c "
import json;d=json.load(open('gpurun_out/bench_final.json'));print('value',d['value'],'ms',d['ms_per_step'],'e2e',d['e2e']['value'],'gapped',d['gapped_stage'],'clk',d['clocks'],'roof',d['roofline'])"
