# GPU pass: parity, bench c2 (with cpu baseline) / heavy / c4 (FPM debug) / c5, launch list c2
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m "gpu and not slow" -x -q --durations=10 > gpurun_out/gputests.log 2>&1; echo rc=$? >> gpurun_out/gputests.log
timeout 400 python bench.py > gpurun_out/bench_c2.json 2> gpurun_out/bench_c2.err
timeout 300 python bench.py --workload heavy --no-cpu-baseline > gpurun_out/bench_heavy.json 2> gpurun_out/bench_heavy.err
GAMMA_DEBUG=1 timeout 900 python bench.py --workload c4 --no-cpu-baseline --steps 3 --warmup 3 > gpurun_out/bench_c4.json 2> gpurun_out/bench_c4.err
timeout 600 python bench.py --workload c5 --steps 2 --warmup 3 > gpurun_out/bench_c5.json 2> gpurun_out/bench_c5.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_c2.csv \
  python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-clocks > /dev/null 2>&1
tail -3 gpurun_out/gputests.log; grep gamma_fpm gpurun_out/bench_c4.err | head; cat gpurun_out/bench_*.json | cut -c1-300
