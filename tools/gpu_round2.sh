#!/bin/bash
# Round evidence: bench line, per-class trace, ncu launch list (time + DRAM bytes) of level-0 sweep 1 on C5
cd "$GRAFT_REPO_ROOT"; mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/smi.txt
timeout 600 python bench.py > gpurun_out/bench_r.jsonl 2> gpurun_out/bench_r.err
timeout 600 python bench.py --impl reference --steps 2 --warmup 3 > gpurun_out/bench_ref.jsonl 2> gpurun_out/bench_ref.err
timeout 900 ncu --profile-from-start off --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct --clock-control none --csv python tools/prof_sweep.py --scale 27 --what sweep1 > gpurun_out/sweep1_launches.csv 2> gpurun_out/ncu1.err
python tools/ncu_table.py gpurun_out/sweep1_launches.csv > gpurun_out/sweep1_launches.txt 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/bench_launches.csv python bench.py --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/bench_ncu.log 2>&1
