#!/bin/bash
# A/B of sweep variants on C5 (LV_TRACE=2 per-class timeline of the second run) + parity of the default
cd "$GRAFT_REPO_ROOT"; mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "sweeps_bit_exact or full_run or alternative or dist_handle" > gpurun_out/ab2_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/ab2_pytest.log
LV_PB=0 timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --e2e-steps 1 --e2e-warmup 0 > gpurun_out/ab2_bench_pb0.jsonl 2>&1
timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --e2e-steps 1 --e2e-warmup 0 > gpurun_out/ab2_bench_pb1.jsonl 2>&1
LV_TRACE=2 timeout 300 python tools/trace_run.py 27 > /dev/null 2> gpurun_out/ab2_trace_pb1.err
for thr in "64,128,256,256,512" "128,128,256,256,512" "64,128,128,256,512" "128,256,256,512,512"; do
  LV_THR=$thr timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --e2e-steps 1 --e2e-warmup 0 > gpurun_out/ab2_bench_thr_${thr//,/_}.jsonl 2>&1
done
