#!/bin/bash
# GPU parity suite (every test, no -x) + the default bench line.
mkdir -p gpurun_out
python -c "from paper_conf_ipps_zhangwlf14_b200 import build; build.build()" > gpurun_out/build.log 2>&1
timeout ${PYTEST_TIMEOUT:-2400} python -m pytest tests -m gpu -q ${PYTEST_ARGS:-} --durations=15 > gpurun_out/pytest_gpu.log 2>&1
echo "pytest rc=$?"; tail -25 gpurun_out/pytest_gpu.log
if [ -z "$NO_BENCH" ]; then
  timeout 900 python bench.py ${BENCH_ARGS:-} > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?"
  cat gpurun_out/bench.json | head -c 3000; tail -5 gpurun_out/bench.err
fi
