# round-1 (session 3) GPU pass: C5 parity + bench lines with §8(d) accounting + per-workload ncu
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
(free -g; nproc; lscpu | head -20) > gpurun_out/host.txt 2>&1
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1200 python -m pytest tests/test_gpu_c5.py -x -q --durations=5 > gpurun_out/c5_test.log 2>&1; echo rc=$? >> gpurun_out/c5_test.log
timeout 400 python bench.py > gpurun_out/bench_c2.json 2> gpurun_out/bench_c2.err
timeout 600 python bench.py --workload c5 --steps 2 --warmup 3 > gpurun_out/bench_c5.json 2> gpurun_out/bench_c5.err
timeout 300 python bench.py --workload heavy --no-cpu-baseline > gpurun_out/bench_heavy.json 2> gpurun_out/bench_heavy.err
# per-workload ncu --set full of the dominant kernels (never a bench number)
timeout 900 ncu --set full --clock-control none --import-source on -k regex:kcl_bitmap -c 4 -o gpurun_out/ncu_c2 -f \
  python bench.py --steps 1 --warmup 0 --no-cpu-baseline --no-clocks > gpurun_out/ncu_c2.log 2>&1
timeout 900 ncu --set full --clock-control none -k regex:kcl_bitmap -c 4 -o gpurun_out/ncu_heavy -f \
  python bench.py --workload heavy --steps 1 --warmup 0 --no-cpu-baseline --no-clocks > gpurun_out/ncu_heavy.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_c2.csv \
  python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-clocks > /dev/null 2>&1
tail -3 gpurun_out/c5_test.log; cat gpurun_out/bench_*.json
