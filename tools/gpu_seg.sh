#!/bin/bash
# Segment-blocked staging: GPU suite, C5 bench A/B (default bits 22, 23, 21, off), serialised trace.
cd "$GRAFT_REPO_ROOT"; mkdir -p gpurun_out; O=gpurun_out/${1:-seg}; mkdir -p $O
timeout 1800 python -m pytest tests -m gpu -q -rs -x > $O/gpu_pytest.log 2>&1; echo "rc=$?" >> $O/gpu_pytest.log
B="python bench.py --steps 5 --warmup 3 --no-cpu-baseline --e2e-steps 1 --e2e-warmup 0"
timeout 600 $B > $O/bench_default.jsonl 2> $O/bench_default.err
LV_SEG=0 timeout 600 $B > $O/bench_seg0.jsonl 2> $O/bench_seg0.err
LV_SEG_BITS=23 timeout 600 $B > $O/bench_b23.jsonl 2> $O/bench_b23.err
LV_SEG_BITS=21 timeout 600 $B > $O/bench_b21.jsonl 2> $O/bench_b21.err
LV_TRACE=2 timeout 300 python tools/trace_run.py 27 > /dev/null 2> $O/trace.err
