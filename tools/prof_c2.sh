#!/bin/bash
# C2 kCL profiling pass (run on the GPU box through gpurun):
#  1. per-|R|-band launch list (GAMMA_KCL_BANDS=1: one warp-team launch per band)
#  2. ncu --set full with source of one warp-team and one CTA-team bitmap launch
# usage: tools/prof_c2.sh [tag]
TAG=${1:-c2}
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python bench.py --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/${TAG}_bench.json 2> gpurun_out/${TAG}_bench.err
GAMMA_KCL_BANDS=1 ncu --metrics gpu__time_duration.sum --clock-control none -c 200 --csv \
  --log-file gpurun_out/${TAG}_bands.csv python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-clocks > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:kcl_bitmap --launch-skip 9 --launch-count 3 \
  -o gpurun_out/${TAG}_full -f python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-clocks > gpurun_out/${TAG}_ncu.log 2>&1
echo done
