#!/bin/bash
# Round-2 check after the cleanup: GPU suite, one bench line, and the per-kernel
# evidence of level-0 sweep 1 on C5: launch list with DRAM bytes, L2 hit rate and
# warp efficiency (active threads per issued instruction), plus ncu --set full
# (source-level) of the table / register kernels.
cd "$GRAFT_REPO_ROOT"; mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r2a_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/r2a_pytest.log
timeout 600 python bench.py > gpurun_out/r2a_bench.jsonl 2> gpurun_out/r2a_bench.err
P="python tools/prof_sweep.py --scale 27 --what sweep1"
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct,smsp__thread_inst_executed_per_inst_executed.ratio,smsp__inst_executed.sum \
  --clock-control none --profile-from-start off --csv --log-file gpurun_out/r2a_sweep1_launches.csv $P > /dev/null 2>&1
NCU="ncu --set full --import-source on --clock-control none --profile-from-start off"
timeout 600 $NCU -k regex:sweep_cta --launch-skip 1 --launch-count 1 -o gpurun_out/r2a_cta $P > /dev/null 2>&1
timeout 600 $NCU -k regex:sweep_small --launch-count 1 -o gpurun_out/r2a_small4 $P > /dev/null 2>&1
timeout 600 $NCU -k regex:k_stage --launch-skip 2 --launch-count 1 -o gpurun_out/r2a_stage_b7 $P > /dev/null 2>&1
timeout 600 $NCU -k regex:sweep_part_stream --launch-count 1 -o gpurun_out/r2a_pstream $P > /dev/null 2>&1
for f in gpurun_out/r2a_*.ncu-rep; do
  ncu -i $f --page details > ${f%.ncu-rep}.details.txt 2>&1
  ncu -i $f --page source --csv --print-source cuda > ${f%.ncu-rep}.src.csv 2>/dev/null
  ncu -i $f --page source --csv > ${f%.ncu-rep}.sass.csv 2>/dev/null
done
