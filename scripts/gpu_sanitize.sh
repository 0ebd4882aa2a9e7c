#!/bin/bash
# compute-sanitizer over scripts/sanitize_cases.py; logs in gpurun_out/sanitizer_<tool>.log
mkdir -p gpurun_out
python -c "from paper_conf_ipps_zhangwlf14_b200 import build; build.build()" > /dev/null 2>&1
for tool in memcheck racecheck synccheck initcheck; do
  extra=""
  [ "$tool" = "memcheck" ] && extra="--leak-check full"
  [ "$tool" = "racecheck" ] && extra="--racecheck-report all"
  timeout ${SAN_TIMEOUT:-1500} compute-sanitizer --tool $tool $extra --print-limit 50 \
     python scripts/sanitize_cases.py ${SAN_ARGS:-quick} > gpurun_out/sanitizer_$tool.log 2>&1
  echo "$tool rc=$? $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY|LEAK SUMMARY' gpurun_out/sanitizer_$tool.log | tr '\n' ' ')"
done
