#!/bin/bash
# ncu --set full of the dominant kernels of one timed step per workload (after 3 warm-up
# steps), plus the launch list of C2 (gpu__time_duration, the bench's own command).
# usage: tools/prof_all.sh   (GPU box; reports land in gpurun_out/)
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
ncu --set full --clock-control none --import-source on -k regex:kcl_bitmap --launch-skip 9 --launch-count 3 \
  -o gpurun_out/prof_c2 -f python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-clocks > gpurun_out/prof_c2.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:kcl_bitmap --launch-skip 6 --launch-count 2 \
  -o gpurun_out/prof_heavy -f python bench.py --workload heavy --steps 1 --warmup 3 --no-cpu-baseline --no-clocks > gpurun_out/prof_heavy.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:sm_kernel --launch-skip 78 --launch-count 26 \
  -o gpurun_out/prof_c3 -f python bench.py --workload c3 --steps 1 --warmup 3 --no-cpu-baseline --no-clocks > gpurun_out/prof_c3.log 2>&1
ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_c2.csv \
  python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-clocks > /dev/null 2>&1
ls -la gpurun_out/prof_*.ncu-rep
