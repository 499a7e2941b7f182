# GPU pass: parity, bench c2/heavy/c3/c4 (FPM debug), ncu c2 + c3 + fpm, launch list c2
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m "gpu and not slow" -x -q --durations=10 > gpurun_out/gputests.log 2>&1; echo rc=$? >> gpurun_out/gputests.log
timeout 400 python bench.py --no-cpu-baseline > gpurun_out/bench_c2.json 2> gpurun_out/bench_c2.err
timeout 300 python bench.py --workload heavy --no-cpu-baseline > gpurun_out/bench_heavy.json 2> gpurun_out/bench_heavy.err
timeout 600 python bench.py --workload c3 --no-cpu-baseline > gpurun_out/bench_c3.json 2> gpurun_out/bench_c3.err
GAMMA_DEBUG=1 timeout 900 python bench.py --workload c4 --no-cpu-baseline --steps 1 --warmup 3 > gpurun_out/bench_c4.json 2> gpurun_out/bench_c4.err
timeout 600 ncu --set full --clock-control none --import-source on -k regex:kcl_bitmap -c 4 -o gpurun_out/ncu_c2f -f \
  python bench.py --steps 1 --warmup 0 --no-cpu-baseline --no-clocks > gpurun_out/ncu_c2f.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_c2.csv \
  python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-clocks > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:sm_ -c 4 -o gpurun_out/ncu_c3f -f \
  python bench.py --workload c3 --steps 1 --warmup 0 --no-cpu-baseline --no-clocks > gpurun_out/ncu_c3f.log 2>&1
timeout 1200 ncu --section SpeedOfLight --section WarpStateStats --section SourceCounters --section MemoryWorkloadAnalysis --section LaunchStats --section Occupancy --metrics dram__bytes_read.sum,dram__bytes_write.sum,smsp__thread_inst_executed_per_inst_executed.ratio --clock-control none --import-source on -k regex:fpm_enum -s 2 -c 1 -o gpurun_out/ncu_c4f -f \
  python bench.py --workload c4 --steps 1 --warmup 0 --no-cpu-baseline --no-clocks > gpurun_out/ncu_c4f.log 2>&1
tail -3 gpurun_out/gputests.log; cat gpurun_out/bench_c4.err | grep gamma_fpm | head; cat gpurun_out/bench_*.json | cut -c1-300
