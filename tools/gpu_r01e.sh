# GPU pass: parity, bench c2/heavy/c5/c4, ncu c2 + heavy bitmap kernels
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m "gpu and not slow" -x -q --durations=10 > gpurun_out/gputests.log 2>&1; echo rc=$? >> gpurun_out/gputests.log
timeout 400 python bench.py > gpurun_out/bench_c2.json 2> gpurun_out/bench_c2.err
timeout 300 python bench.py --workload heavy --no-cpu-baseline > gpurun_out/bench_heavy.json 2> gpurun_out/bench_heavy.err
timeout 600 python bench.py --workload c5 --steps 2 --warmup 3 > gpurun_out/bench_c5.json 2> gpurun_out/bench_c5.err
timeout 900 python bench.py --workload c4 --no-cpu-baseline --steps 3 > gpurun_out/bench_c4.json 2> gpurun_out/bench_c4.err
timeout 600 ncu --set full --clock-control none --import-source on -k regex:kcl_bitmap -c 4 -o gpurun_out/ncu_c2e -f \
  python bench.py --steps 1 --warmup 0 --no-cpu-baseline --no-clocks > gpurun_out/ncu_c2e.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:kcl_bitmap -c 3 -o gpurun_out/ncu_heavye -f \
  python bench.py --workload heavy --steps 1 --warmup 0 --no-cpu-baseline --no-clocks > gpurun_out/ncu_heavye.log 2>&1
tail -3 gpurun_out/gputests.log; cat gpurun_out/bench_*.json | cut -c1-300
