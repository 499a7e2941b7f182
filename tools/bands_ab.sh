cd $GRAFT_REPO_ROOT
for v in 0 1; do
GAMMA_KCL_NO_TABLES=$v GAMMA_KCL_BANDS=1 ncu --metrics gpu__time_duration.sum --clock-control none -c 200 --csv \
  --log-file gpurun_out/bands_t$v.csv python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-clocks > /dev/null 2>&1
done
