#!/bin/bash
# A/B of the working tree (in-tree liblouvain.so) against build/ab/base (tools/ab_build.py) on one
# box: parity files on the new build, then C5 and C3 bench lines alternating base/new twice.
cd "$GRAFT_REPO_ROOT"; mkdir -p gpurun_out; O=gpurun_out/${1:-ab}; mkdir -p $O
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -q -x > $O/pytest.log 2>&1; echo "rc=$?" >> $O/pytest.log
B="python bench.py --steps 5 --warmup 3 --no-cpu-baseline --e2e-steps 1 --e2e-warmup 0"
for r in 1 2; do
  LOUVAIN_LIB=build/ab/base/liblouvain.so timeout 600 $B > $O/C5_base_$r.jsonl 2> $O/C5_base_$r.err
  timeout 600 $B > $O/C5_new_$r.jsonl 2> $O/C5_new_$r.err
done
LOUVAIN_LIB=build/ab/base/liblouvain.so timeout 600 $B --config C3 > $O/C3_base.jsonl 2> $O/C3_base.err
timeout 600 $B --config C3 > $O/C3_new.jsonl 2> $O/C3_new.err
LV_TRACE=2 timeout 300 python tools/trace_run.py 27 > /dev/null 2> $O/trace.err
