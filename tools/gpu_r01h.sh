# GPU pass: parity, all bench lines, ncu captures for profiles/
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,memory.total,clocks.max.sm --format=csv > gpurun_out/smi.txt
timeout 1500 python -m pytest tests -m "gpu and not slow" -x -q --durations=10 > gpurun_out/gputests.log 2>&1; echo rc=$? >> gpurun_out/gputests.log
timeout 400 python bench.py > gpurun_out/bench_c2.json 2> gpurun_out/bench_c2.err
timeout 300 python bench.py --workload c1 > gpurun_out/bench_c1.json 2> gpurun_out/bench_c1.err
timeout 300 python bench.py --workload heavy --no-cpu-baseline > gpurun_out/bench_heavy.json 2> gpurun_out/bench_heavy.err
timeout 600 python bench.py --workload c3 --no-cpu-baseline > gpurun_out/bench_c3.json 2> gpurun_out/bench_c3.err
GAMMA_DEBUG=1 timeout 900 python bench.py --workload c4 --no-cpu-baseline --steps 3 --warmup 3 > gpurun_out/bench_c4.json 2> gpurun_out/bench_c4.err
timeout 600 python bench.py --workload c5 --steps 2 --warmup 3 > gpurun_out/bench_c5.json 2> gpurun_out/bench_c5.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_c2.csv \
  python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-clocks > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:kcl_bitmap -c 4 -o gpurun_out/ncu_c2 -f \
  python bench.py --steps 1 --warmup 0 --no-cpu-baseline --no-clocks > gpurun_out/ncu_c2.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:kcl_bitmap -c 3 -o gpurun_out/ncu_heavy -f \
  python bench.py --workload heavy --steps 1 --warmup 0 --no-cpu-baseline --no-clocks > gpurun_out/ncu_heavy.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:sm_kernel -c 12 -o gpurun_out/ncu_c3 -f \
  python bench.py --workload c3 --steps 1 --warmup 0 --no-cpu-baseline --no-clocks > gpurun_out/ncu_c3.log 2>&1
timeout 1200 ncu --section SpeedOfLight --section WarpStateStats --section SourceCounters --section MemoryWorkloadAnalysis --section LaunchStats --section Occupancy --metrics dram__bytes_read.sum,dram__bytes_write.sum,smsp__thread_inst_executed_per_inst_executed.ratio,lts__t_sector_hit_rate.pct,sm__inst_issued.avg.pct_of_peak_sustained_active,sm__warps_active.avg.pct_of_peak_sustained_active,smsp__inst_executed.sum,l1tex__t_sector_hit_rate.pct,launch__registers_per_thread,launch__grid_size,gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed,sm__throughput.avg.pct_of_peak_sustained_elapsed --clock-control none --import-source on -k regex:fpm_enum -s 2 -c 1 -o gpurun_out/ncu_c4 -f \
  python bench.py --workload c4 --steps 1 --warmup 0 --no-cpu-baseline --no-clocks > gpurun_out/ncu_c4.log 2>&1
tail -3 gpurun_out/gputests.log; grep gamma_fpm gpurun_out/bench_c4.err | head -4; cat gpurun_out/bench_*.json | cut -c1-250
