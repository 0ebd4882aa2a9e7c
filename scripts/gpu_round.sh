#!/bin/bash
# Full GPU check: tests, bench (config 3), per-kernel ncu roofline, strategy sweep.
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -x --durations=8 > gpurun_out/pytest_gpu.log 2>&1
tail -12 gpurun_out/pytest_gpu.log
timeout 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?"
cat gpurun_out/bench.json
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,sm__throughput.avg.pct_of_peak_sustained_elapsed \
  --clock-control none --csv --log-file gpurun_out/kernels.csv python scripts/kernel_roofline.py run > gpurun_out/kernels.log 2>&1
echo "ncu kernels rc=$?"
python scripts/kernel_roofline.py summarize gpurun_out/kernels.csv gpurun_out/kernels.json
timeout 900 python scripts/sweep.py gpurun_out/sweep.json 5 > gpurun_out/sweep.txt 2>&1; echo "sweep rc=$?"
cat gpurun_out/sweep.txt | tail -30
