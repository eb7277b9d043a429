#!/bin/bash
# A/B of the stage/table pipeline (LV_PIPE=0 vs on, stage CTAs per SM), parity of the default
cd "$GRAFT_REPO_ROOT"; mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q > gpurun_out/ab4_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/ab4_pytest.log
B="python bench.py --steps 5 --warmup 3 --no-cpu-baseline --e2e-steps 1 --e2e-warmup 0"
LV_PIPE=0 timeout 300 $B > gpurun_out/ab4_pipe0.jsonl 2>&1
timeout 300 $B > gpurun_out/ab4_pipe_sm4.jsonl 2>&1
LV_STAGE_SM=2 timeout 300 $B > gpurun_out/ab4_pipe_sm2.jsonl 2>&1
LV_STAGE_SM=8 timeout 300 $B > gpurun_out/ab4_pipe_sm8.jsonl 2>&1
LV_PIPE=0 timeout 300 $B --config C3 > gpurun_out/ab4_c3_pipe0.jsonl 2>&1
timeout 300 $B --config C3 > gpurun_out/ab4_c3_pipe_sm4.jsonl 2>&1
