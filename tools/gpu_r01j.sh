# GPU pass (session 4b): induced-SM parity, bench lines, launch list + ncu summaries (summarised
# on the box; .ncu-rep files removed so gpurun_out stays under the 64 MiB copy-back limit), ablation
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/prof
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke rc=$? >> gpurun_out/smoke.log
timeout 900 python -m pytest tests/test_gpu_match.py tests/test_plan.py -q > gpurun_out/gputests_match.log 2>&1; echo rc=$? >> gpurun_out/gputests_match.log
timeout 400 python bench.py > gpurun_out/bench_c2.json 2> gpurun_out/bench_c2.err
timeout 300 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/bench_ref.json 2> gpurun_out/bench_ref.err
timeout 300 python bench.py --workload c1 > gpurun_out/bench_c1.json 2> gpurun_out/bench_c1.err
timeout 300 python bench.py --workload heavy --no-cpu-baseline > gpurun_out/bench_heavy.json 2> gpurun_out/bench_heavy.err
timeout 600 python bench.py --workload c3 --no-cpu-baseline > gpurun_out/bench_c3.json 2> gpurun_out/bench_c3.err
timeout 900 python bench.py --workload c4 --no-cpu-baseline --steps 3 --warmup 3 > gpurun_out/bench_c4.json 2> gpurun_out/bench_c4.err
timeout 900 python bench.py --workload c5 --steps 2 --warmup 3 > gpurun_out/bench_c5.json 2> gpurun_out/bench_c5.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_c2.csv \
  python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-clocks > /dev/null 2>&1
python tools/launch_summary.py gpurun_out/launches_c2.csv gpurun_out/prof/launches_c2_r01.md "ncu --metrics gpu__time_duration.sum --clock-control none --csv python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-clocks"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_c3.csv \
  python bench.py --workload c3 --steps 1 --warmup 1 --no-cpu-baseline --no-clocks > /dev/null 2>&1
python tools/launch_summary.py gpurun_out/launches_c3.csv gpurun_out/prof/launches_c3_r01.md "ncu ... python bench.py --workload c3 --steps 1 --warmup 1"
rm -f gpurun_out/launches_c2.csv gpurun_out/launches_c3.csv
timeout 900 ncu --set full --clock-control none --import-source on -k regex:kcl_bitmap -c 3 -o /tmp/ncu_c2 -f \
  python bench.py --steps 1 --warmup 0 --no-cpu-baseline --no-clocks > gpurun_out/ncu_c2.log 2>&1
python tools/ncu_summary.py /tmp/ncu_c2.ncu-rep gpurun_out/prof r01 c2 >> gpurun_out/ncu_c2.log 2>&1
ncu -i /tmp/ncu_c2.ncu-rep --page source --csv > /tmp/src_c2.csv 2>/dev/null; gzip -c /tmp/src_c2.csv > gpurun_out/src_c2_sass.csv.gz
timeout 900 ncu --set full --clock-control none --import-source on -k regex:sm_kernel -c 6 -o /tmp/ncu_c3 -f \
  python bench.py --workload c3 --steps 1 --warmup 0 --no-cpu-baseline --no-clocks > gpurun_out/ncu_c3.log 2>&1
python tools/ncu_summary.py /tmp/ncu_c3.ncu-rep gpurun_out/prof r01 c3 >> gpurun_out/ncu_c3.log 2>&1
timeout 900 python tools/ablation.py > gpurun_out/ablation.jsonl 2> gpurun_out/ablation.err
du -sh gpurun_out
tail -3 gpurun_out/gputests_match.log; tail -1 gpurun_out/smoke.log; cat gpurun_out/bench_*.json | cut -c1-200
