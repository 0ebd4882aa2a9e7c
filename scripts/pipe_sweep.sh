#!/bin/bash
# e2e pipeline shape on config 3: H2D rate, then blastp_search_host_db with
# automatic parts (growth knob) and fixed part counts.
mkdir -p gpurun_out
timeout 300 python scripts/h2d_probe.py 2>&1 | head -8
for g in 150 125 110; do
  echo "growth $g"; BLASTP_PIPE_GROWTH=$g timeout 300 python scripts/pipe_probe.py 1.0 0 2>/dev/null | tail -2
done
for n in 8 16 32; do
  echo "parts $n"; timeout 300 python scripts/pipe_probe.py 1.0 $n 2>/dev/null | tail -2
done
