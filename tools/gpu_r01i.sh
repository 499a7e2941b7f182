# GPU pass (session 4): full -m gpu suite incl. slow, smoke, all bench lines, launch list + ncu full of c2 bitmap kernel
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,memory.total,clocks.max.sm --format=csv > gpurun_out/smi.txt
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke rc=$? >> gpurun_out/smoke.log
timeout 2400 python -m pytest tests -m gpu -q --durations=15 > gpurun_out/gputests.log 2>&1; echo rc=$? >> gpurun_out/gputests.log
timeout 400 python bench.py > gpurun_out/bench_c2.json 2> gpurun_out/bench_c2.err
timeout 300 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/bench_ref.json 2> gpurun_out/bench_ref.err
timeout 300 python bench.py --workload c1 > gpurun_out/bench_c1.json 2> gpurun_out/bench_c1.err
timeout 300 python bench.py --workload heavy --no-cpu-baseline > gpurun_out/bench_heavy.json 2> gpurun_out/bench_heavy.err
timeout 600 python bench.py --workload c3 --no-cpu-baseline > gpurun_out/bench_c3.json 2> gpurun_out/bench_c3.err
GAMMA_DEBUG=1 timeout 900 python bench.py --workload c4 --no-cpu-baseline --steps 3 --warmup 3 > gpurun_out/bench_c4.json 2> gpurun_out/bench_c4.err
timeout 900 python bench.py --workload c5 --steps 2 --warmup 3 > gpurun_out/bench_c5.json 2> gpurun_out/bench_c5.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_c2.csv \
  python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-clocks > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:kcl_bitmap -c 4 -o gpurun_out/ncu_c2 -f \
  python bench.py --steps 1 --warmup 0 --no-cpu-baseline --no-clocks > gpurun_out/ncu_c2.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:sm_kernel -c 12 -o gpurun_out/ncu_c3 -f \
  python bench.py --workload c3 --steps 1 --warmup 0 --no-cpu-baseline --no-clocks > gpurun_out/ncu_c3.log 2>&1
tail -3 gpurun_out/gputests.log; cat gpurun_out/smoke.log | tail -2; cat gpurun_out/bench_*.json | cut -c1-250
