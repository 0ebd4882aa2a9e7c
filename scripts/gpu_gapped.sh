#!/bin/bash
# Gapped-stage iteration: build, its parity tests, a timing of the stage on config 3.
mkdir -p gpurun_out
python -c "from paper_conf_ipps_zhangwlf14_b200 import build; build.build()" > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
timeout ${PYTEST_TIMEOUT:-1500} python -m pytest tests/test_gpu_gapped.py -m gpu -q -x ${PYTEST_K:+-k "$PYTEST_K"} --durations=8 > gpurun_out/pytest_gapped.log 2>&1
echo "pytest rc=$?"; tail -40 gpurun_out/pytest_gapped.log
if [ -f scripts/gapped_time.py ]; then PYTHONPATH=. timeout 900 python scripts/gapped_time.py > gpurun_out/gapped_time.txt 2>&1; echo "time rc=$?"; cat gpurun_out/gapped_time.txt; fi
