#!/bin/bash
# Full GPU suite + bench lines of every BASELINE.json config + oracle timing on the box's host
cd "$GRAFT_REPO_ROOT"; mkdir -p gpurun_out
timeout 1800 python -m pytest tests -m gpu -q -rs > gpurun_out/r2d_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/r2d_pytest.log
timeout 900 python bench.py > gpurun_out/r2d_bench_C5.jsonl 2> gpurun_out/r2d_bench_C5.err
for c in C1 C2 C3 C4a C4b; do
  timeout 600 python bench.py --config $c --steps 10 --warmup 3 > gpurun_out/r2d_bench_$c.jsonl 2> gpurun_out/r2d_bench_$c.err
done
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/r2d_ref_C5.jsonl 2> gpurun_out/r2d_ref_C5.err
for c in C2 C3; do timeout 900 python tools/oracle_timing.py $c --full > gpurun_out/r2d_oracle_timing_$c.json 2>&1; done
timeout 1500 python tools/oracle_timing.py C5 > gpurun_out/r2d_oracle_timing_C5.json 2>&1
