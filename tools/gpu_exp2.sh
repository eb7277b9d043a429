#!/bin/bash
cd "$GRAFT_REPO_ROOT"; mkdir -p gpurun_out
LV_TRACE=2 timeout 600 python tools/relabel_exp.py --scale 27 --mode both > gpurun_out/exp2_cs.out 2> gpurun_out/exp2_cs.err
LV_STAGE_WB=1 LV_TRACE=2 timeout 600 python tools/relabel_exp.py --scale 27 --mode natural > gpurun_out/exp2_wb.out 2> gpurun_out/exp2_wb.err
