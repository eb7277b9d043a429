#!/bin/bash
# One gpurun call: GPU tests, bench, per-level/per-class trace, ncu launch list of sweep 1.
cd "$GRAFT_REPO_ROOT"
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/smi.txt
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 600 python bench.py > gpurun_out/bench.jsonl 2> gpurun_out/bench.err
LV_TRACE=2 timeout 300 python tools/trace_run.py 27 > gpurun_out/trace.out 2> gpurun_out/trace.err
timeout 900 ncu --profile-from-start off --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct --clock-control none --csv python tools/prof_sweep.py --scale 27 --what sweep1 > gpurun_out/sweep1_launches.csv 2> gpurun_out/ncu1.err
python tools/ncu_table.py gpurun_out/sweep1_launches.csv > gpurun_out/sweep1_launches.txt 2>&1
