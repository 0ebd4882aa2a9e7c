#!/bin/bash
# e2e pipeline shape on config 3: blastp_search_host_db with one / two search
# streams, automatic parts (growth knob) and fixed part counts.
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "host_db" 2>&1 | tail -2
for st in 1 2; do
  for g in 150 125; do
    echo "streams $st growth $g"; BLASTP_PIPE_STREAMS=$st BLASTP_PIPE_GROWTH=$g timeout 300 python scripts/pipe_probe.py 1.0 0 2>/dev/null | tail -1
  done
  for n in 8 16 32; do
    echo "streams $st parts $n"; BLASTP_PIPE_STREAMS=$st timeout 300 python scripts/pipe_probe.py 1.0 $n 2>/dev/null | tail -1
  done
done
