#!/bin/bash
# Round evidence on one B200: GPU suite, smoke, bench lines of every config + reference arm, the
# N > 1 path (2 ranks sharing the GPU, both exchange modes), sweep-1 launch list with DRAM bytes /
# L2 hit / warp efficiency, the bench command's launch list, ncu --set full of the top kernels.
cd "$GRAFT_REPO_ROOT"; mkdir -p gpurun_out; O=gpurun_out/final; mkdir -p $O
timeout 1800 python -m pytest tests -m gpu -q -rs > $O/gpu_pytest.log 2>&1; echo "rc=$?" >> $O/gpu_pytest.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > $O/smoke.log 2>&1
timeout 900 python bench.py > $O/bench_C5.jsonl 2> $O/bench_C5.err
for c in C1 C2 C3 C4a C4b; do
  timeout 600 python bench.py --config $c --steps 10 --warmup 3 > $O/bench_$c.jsonl 2> $O/bench_$c.err
done
timeout 900 python bench.py --impl reference --steps 3 --warmup 3 > $O/bench_C5_reference.jsonl 2> $O/bench_C5_reference.err
for x in allgather p2p; do
  LV_BENCH_ONE_GPU=1 timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 \
    --master-port 29533 bench.py --gpus 2 --steps 2 --warmup 1 --config C2 --backend gloo --exchange $x --e2e-steps 1 \
    > $O/bench_dist2_C2_$x.jsonl 2> $O/bench_dist2_C2_$x.err
done
P="python tools/prof_sweep.py --scale 27 --what sweep1"
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct,smsp__thread_inst_executed_per_inst_executed.ratio,smsp__inst_executed.sum \
  --clock-control none --profile-from-start off --csv --log-file $O/sweep1_launches.csv $P > /dev/null 2>&1
timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/bench_launches.csv \
  python bench.py --steps 1 --warmup 1 --no-cpu-baseline --e2e-steps 1 --e2e-warmup 0 > /dev/null 2>&1
NCU="ncu --set full --import-source on --clock-control none --profile-from-start off"
timeout 600 $NCU -k regex:k_stage --launch-skip 1 --launch-count 1 -o $O/ncu_stage $P > /dev/null 2>&1
timeout 600 $NCU -k regex:sweep_cta_c --launch-skip 1 --launch-count 1 -o $O/ncu_cta $P > /dev/null 2>&1
timeout 600 $NCU -k regex:sweep_part_stream --launch-count 1 -o $O/ncu_pstream $P > /dev/null 2>&1
timeout 600 $NCU -k regex:sweep_small --launch-count 1 -o $O/ncu_small $P > /dev/null 2>&1
timeout 600 $NCU -k regex:sweep_warp_d --launch-count 1 -o $O/ncu_warpd $P > /dev/null 2>&1
for f in $O/ncu_*.ncu-rep; do
  ncu -i $f --page details > ${f%.ncu-rep}.details.txt 2>&1
  ncu -i $f --page source --csv > ${f%.ncu-rep}.sass.csv 2>/dev/null
done
