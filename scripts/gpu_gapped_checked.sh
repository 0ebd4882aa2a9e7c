#!/bin/bash
# The gapped-stage tests on the product build and on a bounds-checked build
# (-DGAPPED_CHECK: device asserts on every sequence read and store index;
# compute-sanitizer is closed on this pool).
mkdir -p gpurun_out
python -c "from paper_conf_ipps_zhangwlf14_b200 import build; build.build()" > /dev/null 2>&1 || exit 1
[ -f ab/check.so ] || bash scripts/build_variant.sh check -DGAPPED_CHECK > /dev/null
python -m pytest tests/test_gpu_gapped.py -m gpu -q -x 2>&1 | tail -2
BLASTP_LIB=$PWD/ab/check.so python -m pytest tests/test_gpu_gapped.py -m gpu -q -x 2>&1 | tail -2
