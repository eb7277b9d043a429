#!/bin/bash
cd "$GRAFT_REPO_ROOT"; mkdir -p gpurun_out
LV_TRACE=2 timeout 600 python tools/relabel_exp.py --scale 27 --mode both > gpurun_out/relabel.out 2> gpurun_out/relabel.err
LV_L2WIN=100000000 LV_TRACE=2 timeout 600 python tools/relabel_exp.py --scale 27 --mode relabel > gpurun_out/relabel_win.out 2> gpurun_out/relabel_win.err
LV_TRACE=1 LV_CONTRACT=hash timeout 600 python tools/trace_run.py 27 > gpurun_out/trace_hash.out 2> gpurun_out/trace_hash.err
