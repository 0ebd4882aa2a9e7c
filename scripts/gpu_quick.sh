#!/bin/bash
# Quick GPU iteration: build, a parity subset on one kernel variant, a short bench.
mkdir -p gpurun_out
python -c "from paper_conf_ipps_zhangwlf14_b200 import build; build.build()" > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
timeout ${PYTEST_TIMEOUT:-900} python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "${PYTEST_K:-block}" --durations=5 > gpurun_out/pytest_quick.log 2>&1
echo "pytest rc=$?"; tail -30 gpurun_out/pytest_quick.log
timeout 600 python bench.py --steps 20 --warmup 3 --no-cpu-baseline --no-e2e ${BENCH_ARGS:-} > gpurun_out/bench_quick.json 2> gpurun_out/bench_quick.err; echo "bench rc=$?"
python -c "
import json;d=json.load(open('gpurun_out/bench_quick.json'));print('value',d['value'],'ms',d['ms_per_step'],'hsps',d['config']['hsps_per_step'],'clk',d['clocks'])" ; tail -3 gpurun_out/bench_quick.err
