#!/bin/bash
# the N > 1 bench path (run_sharded_bench) with 2 ranks on one GPU over gloo, on R-MAT s20 (diagnostics only)
cd "$GRAFT_REPO_ROOT"; mkdir -p gpurun_out
LV_BENCH_ONE_GPU=1 timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29531 bench.py --gpus 2 --steps 2 --warmup 3 --scale 20 --backend gloo > gpurun_out/bench_dist2.jsonl 2> gpurun_out/bench_dist2.err; echo "rc=$?" >> gpurun_out/bench_dist2.err
