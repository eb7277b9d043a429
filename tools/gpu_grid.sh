cd "$GRAFT_REPO_ROOT"; mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -k threshold_grid -q > gpurun_out/grid_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/grid_pytest.log
timeout 1500 python tools/threshold_grid.py C3 C4a C4b C5 C2 > gpurun_out/threshold_grid.jsonl 2> gpurun_out/threshold_grid.err
