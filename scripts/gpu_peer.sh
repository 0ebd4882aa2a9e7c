#!/bin/bash
# The fused search + gather (PeerHspBuffer): its parity tests, then a 2-rank
# bench on the one GPU (gloo host collectives, CUDA IPC on the same device)
# with --gather p2p and --gather nccl.
mkdir -p gpurun_out
python -c "from paper_conf_ipps_zhangwlf14_b200 import build; build.build()" > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_peer.py tests/test_bench_contract.py -m gpu -q -x --durations=5 > gpurun_out/pytest_peer.log 2>&1
echo "pytest rc=$?"; tail -15 gpurun_out/pytest_peer.log
for g in p2p nccl; do
  BLASTP_DIST_BACKEND=gloo timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 \
    --master-addr 127.0.0.1 --master-port 29517 bench.py --gpus 2 --steps 3 --warmup 3 --no-e2e \
    --gather $g > gpurun_out/bench_2rank_$g.json 2> gpurun_out/bench_2rank_$g.err
  echo "2-rank $g rc=$?"; head -c 600 gpurun_out/bench_2rank_$g.json; echo; tail -3 gpurun_out/bench_2rank_$g.err
done
