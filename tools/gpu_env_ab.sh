#!/bin/bash
# Env-knob A/B on one box and one build: C5 bench lines alternating default / each "K=V" given,
# twice, plus a serialised trace per setting.  Usage: gpu_env_ab.sh NAME "K=V" ["K2=V2" ...]
cd "$GRAFT_REPO_ROOT"; mkdir -p gpurun_out; O=gpurun_out/$1; shift; mkdir -p $O
B="python bench.py --steps 5 --warmup 3 --no-cpu-baseline --e2e-steps 1 --e2e-warmup 0"
for r in 1 2; do
  timeout 600 $B > $O/C5_default_$r.jsonl 2> $O/C5_default_$r.err
  for kv in "$@"; do env $kv timeout 600 $B > $O/C5_${kv}_$r.jsonl 2> $O/C5_${kv}_$r.err; done
done
LV_TRACE=2 timeout 300 python tools/trace_run.py 27 > /dev/null 2> $O/trace_default.err
for kv in "$@"; do env $kv LV_TRACE=2 timeout 300 python tools/trace_run.py 27 > /dev/null 2> $O/trace_${kv}.err; done
