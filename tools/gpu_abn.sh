#!/bin/bash
# Same-box A/B of several builds: gpu_abn.sh OUT NAME... (NAME = a build/ab/NAME/liblouvain.so
# from tools/ab_build.py, or "tree" for the in-tree library).  C5 bench lines, the variants
# alternating, twice; then a serialised trace of each; parity files on each non-tree build.
cd "$GRAFT_REPO_ROOT"; mkdir -p gpurun_out; O=gpurun_out/$1; shift; mkdir -p $O
lib() { [ "$1" = tree ] && echo "" || echo "build/ab/$1/liblouvain.so"; }
B="python bench.py --steps 5 --warmup 3 --no-cpu-baseline --e2e-steps 1 --e2e-warmup 0"
for v in "$@"; do
  if [ "$v" != tree ] && [ -z "$ABN_NOTEST" ]; then
    LOUVAIN_LIB=$(lib $v) timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -q -x \
      > $O/pytest_$v.log 2>&1; echo "rc=$?" >> $O/pytest_$v.log
  fi
done
for r in 1 2; do
  for v in "$@"; do LOUVAIN_LIB=$(lib $v) timeout 600 $B > $O/C5_${v}_$r.jsonl 2> $O/C5_${v}_$r.err; done
done
for v in "$@"; do LOUVAIN_LIB=$(lib $v) LV_TRACE=2 timeout 300 python tools/trace_run.py 27 > /dev/null 2> $O/trace_$v.err; done
