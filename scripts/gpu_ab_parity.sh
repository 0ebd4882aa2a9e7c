#!/bin/bash
# A/B of ab/*.so builds (scripts/ab_kernel.py), then the block-kernel parity
# subset with ab/$PARITY.so installed as the library (no rebuild: newer than
# the sources).  usage: PARITY=name bash scripts/gpu_ab_parity.sh a.so b.so ...
mkdir -p gpurun_out
timeout 900 python scripts/ab_kernel.py ${AB_ROUNDS:-6} "$@" 2>&1 | tail -${AB_TAIL:-12}
if [ -n "$PARITY" ]; then
  cp ab/$PARITY.so paper_conf_ipps_zhangwlf14_b200/libblastp.so
  touch paper_conf_ipps_zhangwlf14_b200/libblastp.so
  timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_stateful.py -m gpu -q -x \
    -k "${PYTEST_K:-block}" > gpurun_out/pytest_ab_parity.log 2>&1
  echo "parity($PARITY) rc=$?"; tail -5 gpurun_out/pytest_ab_parity.log
fi
