#!/bin/bash
# Short device-only bench of kernel variants / knobs (config 3, 10 steps).
mkdir -p gpurun_out
run() { echo "== $*"; env "$@" timeout 600 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline ${BENCH_ARGS:-} 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(f\"   ms/step {d['ms_per_step']:.2f}  value {d['value']:.4g}\")"; }
for v in "${@:-BLASTP_KERNEL=warp}"; do run $v; done
