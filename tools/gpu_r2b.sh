#!/bin/bash
# Distributed handle check: GPU suite (incl. the dist-handle parity tests), the N > 1 bench
# path with 2 ranks on one GPU (host transport over gloo), and a per-class trace of a C5 run.
cd "$GRAFT_REPO_ROOT"; mkdir -p gpurun_out
timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/r2b_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/r2b_pytest.log
LV_BENCH_ONE_GPU=1 timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 \
  --master-port 29533 bench.py --gpus 2 --steps 2 --warmup 1 --config C3 --backend gloo --e2e-steps 1 \
  > gpurun_out/r2b_bench_dist2.jsonl 2> gpurun_out/r2b_bench_dist2.err
LV_TRACE=2 timeout 600 python tools/trace_run.py 27 > /dev/null 2> gpurun_out/r2b_trace_c5.err
