#!/bin/bash
# Distributed handle with sharded contraction: parity (2-3 ranks share the GPU) + the N>1 bench path
cd "$GRAFT_REPO_ROOT"; mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_parity.py -x -q -k "dist_handle or loaded_files or alternative" > gpurun_out/r2c_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/r2c_pytest.log
LV_BENCH_ONE_GPU=1 timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 \
  --master-port 29533 bench.py --gpus 2 --steps 2 --warmup 1 --config C3 --backend gloo --e2e-steps 1 \
  > gpurun_out/r2c_bench_dist2.jsonl 2> gpurun_out/r2c_bench_dist2.err
timeout 600 python bench.py --config C3 --steps 3 --warmup 3 > gpurun_out/r2c_bench_c3.jsonl 2> gpurun_out/r2c_bench_c3.err
