#!/bin/bash
# e2e (formatted host DB streamed per step) under part-plan knobs, config 3.
mkdir -p gpurun_out
python -c "from paper_conf_ipps_zhangwlf14_b200 import build; build.build()" > gpurun_out/build.log 2>&1 || exit 1
for cfg in ${PIPE_CFGS:-"" "BLASTP_PIPE_GROWTH=150" "BLASTP_PIPE_GROWTH=120" "BLASTP_PIPE_GROWTH=130"}; do
  env $cfg timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --e2e-steps 5 > gpurun_out/pipe.json 2>/dev/null
  python -c "
import json;d=json.load(open('gpurun_out/pipe.json'));e=d['e2e']
print('$cfg'.ljust(50), 'dev %.2f ms'%d['ms_per_step'], 'e2e %.2f ms parts %d'%(e['ms_per_step'],e['parts']), 'ascii %.2f'%d['e2e_ascii_db']['ms_per_step'])"
done
