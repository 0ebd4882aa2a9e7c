#!/bin/bash
# Round-end GPU evidence: build, smoke(), the whole -m gpu suite (log kept).
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?"; tail -2 gpurun_out/smoke.log
timeout ${SUITE_TIMEOUT:-3000} python -m pytest tests -m gpu -q -x --durations=15 > gpurun_out/pytest_gpu_full.log 2>&1
echo "pytest rc=$?"; tail -25 gpurun_out/pytest_gpu_full.log
