#!/bin/bash
# Re-entry check of HEAD: GPU suite, smoke, C5 bench line, serialised per-step trace of a C5 run,
# and the launch list of one bench run (kernel shares).
cd "$GRAFT_REPO_ROOT"; mkdir -p gpurun_out; O=gpurun_out/${1:-r2f}; mkdir -p $O
timeout 1800 python -m pytest tests -m gpu -q -rs -x > $O/gpu_pytest.log 2>&1; echo "rc=$?" >> $O/gpu_pytest.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > $O/smoke.log 2>&1
timeout 900 python bench.py > $O/bench_C5.jsonl 2> $O/bench_C5.err
LV_TRACE=2 timeout 300 python tools/trace_run.py 27 > /dev/null 2> $O/trace.err
timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/bench_launches.csv \
  python bench.py --steps 1 --warmup 1 --no-cpu-baseline --e2e-steps 1 --e2e-warmup 0 > /dev/null 2>&1
