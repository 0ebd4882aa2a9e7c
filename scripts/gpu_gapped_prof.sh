#!/bin/bash
# Gapped stage: config-3 parity, a launch list of the stage and full captures
# of its two DP kernels.
mkdir -p gpurun_out
python -c "from paper_conf_ipps_zhangwlf14_b200 import build; build.build()" > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
if [ -z "${SKIP_PARITY:-}" ]; then
timeout 1500 python -m pytest tests/test_gpu_gapped.py -m gpu -q -x -k config3 --durations=3 > gpurun_out/pytest_gapped_c3.log 2>&1
echo "pytest rc=$?"; tail -8 gpurun_out/pytest_gapped_c3.log
fi
PYTHONPATH=. timeout 600 python scripts/gapped_time.py ${TIME_ARGS:-} > gpurun_out/gapped_time.txt 2>&1; echo "time rc=$?"; cat gpurun_out/gapped_time.txt
PYTHONPATH=. timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv -k regex:gapped \
  --log-file gpurun_out/gapped_launches.csv python scripts/gapped_time.py > /dev/null 2>&1; echo "ncu list rc=$?"
PYTHONPATH=. timeout 1500 ncu --set full --clock-control none --import-source on -k regex:"gapped_(score|trace)" \
  -c 2 -o gpurun_out/prof_gapped python scripts/gapped_time.py > gpurun_out/ncu_gapped.log 2>&1; echo "ncu full rc=$?"
tail -3 gpurun_out/ncu_gapped.log
