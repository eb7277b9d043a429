#!/bin/bash
cd "$GRAFT_REPO_ROOT"; mkdir -p gpurun_out
timeout 600 python bench.py > gpurun_out/bench13.jsonl 2> gpurun_out/bench13.err
LV_OVERLAP=0 timeout 600 python bench.py > gpurun_out/bench13_serial.jsonl 2> gpurun_out/bench13_serial.err
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_ab13.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_ab13.log
