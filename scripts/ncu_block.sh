#!/bin/bash
# One full ncu capture of the search kernel on config 3 (+ launch list of a short bench).
mkdir -p gpurun_out
python -c "from paper_conf_ipps_zhangwlf14_b200 import build; build.build()" > gpurun_out/build.log 2>&1 || exit 1
K=${KREGEX:-search_}
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:$K -s 1 -c 1 \
  -o gpurun_out/${PROF:-prof_block} -f python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline ${BENCH_ARGS:-} > gpurun_out/ncu_full.log 2>&1
echo "ncu rc=$?"; tail -3 gpurun_out/ncu_full.log
