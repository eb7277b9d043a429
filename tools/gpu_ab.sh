#!/bin/bash
# A/B of a path-selection variable: parity suites on the default, then C5 and C3 bench lines
# with and without "$1=$2", and a per-class trace of a C5 run.  Usage: gpu_ab.sh VAR VALUE TAG
cd "$GRAFT_REPO_ROOT"; mkdir -p gpurun_out
V=$1; X=$2; T=${3:-ab}
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -x -q > gpurun_out/${T}_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/${T}_pytest.log
B="python bench.py --no-cpu-baseline --e2e-steps 1 --e2e-warmup 0"
for c in C5 C3; do
  timeout 600 $B --config $c --steps 5 --warmup 3 > gpurun_out/${T}_${c}_default.jsonl 2>&1
  env $V=$X timeout 600 $B --config $c --steps 5 --warmup 3 > gpurun_out/${T}_${c}_${V}.jsonl 2>&1
done
LV_TRACE=1 timeout 300 python tools/trace_run.py 27 > /dev/null 2> gpurun_out/${T}_trace.err
