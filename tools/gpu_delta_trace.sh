cd "$GRAFT_REPO_ROOT"; mkdir -p gpurun_out
LV_TRACE=1 timeout 300 python tools/trace_run.py 27 > /dev/null 2> gpurun_out/delta_trace.err
LV_MOD_DELTA=0 LV_TRACE=1 timeout 300 python tools/trace_run.py 27 > /dev/null 2> gpurun_out/delta_trace_off.err
