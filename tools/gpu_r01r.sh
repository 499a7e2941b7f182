# GPU pass (session 5f): refreshed round-1 numbers after the SM long-child probe: smoke, full
# -m gpu suite, bench lines c1..c5/heavy/reference, launch lists + ncu --set full for c2 and c3
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/r/prof
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/r/smoke.log 2>&1; echo smoke rc=$? >> gpurun_out/r/smoke.log
timeout 400 python bench.py > gpurun_out/r/bench_c2.json 2> gpurun_out/r/bench_c2.err
timeout 300 python bench.py --workload c1 > gpurun_out/r/bench_c1.json 2> gpurun_out/r/bench_c1.err
timeout 300 python bench.py --workload heavy --no-cpu-baseline > gpurun_out/r/bench_heavy.json 2> gpurun_out/r/bench_heavy.err
timeout 600 python bench.py --workload c3 --no-cpu-baseline > gpurun_out/r/bench_c3.json 2> gpurun_out/r/bench_c3.err
timeout 900 python bench.py --workload c4 --no-cpu-baseline --steps 3 --warmup 3 > gpurun_out/r/bench_c4.json 2> gpurun_out/r/bench_c4.err
timeout 900 python bench.py --workload c5 --steps 2 --warmup 3 > gpurun_out/r/bench_c5.json 2> gpurun_out/r/bench_c5.err
timeout 300 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/r/bench_ref.json 2> gpurun_out/r/bench_ref.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file /tmp/launches_c3.csv \
  python bench.py --workload c3 --steps 1 --warmup 1 --no-cpu-baseline --no-clocks > /dev/null 2>&1
python tools/launch_summary.py /tmp/launches_c3.csv gpurun_out/r/prof/launches_c3_r01.md "ncu --metrics gpu__time_duration.sum --clock-control none --csv python bench.py --workload c3 --steps 1 --warmup 1 --no-cpu-baseline --no-clocks"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:sm_kernel -s 6 -c 8 -o /tmp/ncu_c3 -f \
  python bench.py --workload c3 --steps 1 --warmup 0 --no-cpu-baseline --no-clocks > gpurun_out/r/ncu_c3.log 2>&1
python tools/ncu_summary.py /tmp/ncu_c3.ncu-rep gpurun_out/r/prof r01 c3 >> gpurun_out/r/ncu_c3.log 2>&1
cp /tmp/ncu_c3.ncu-rep gpurun_out/r/ 2>/dev/null
timeout 1800 python -m pytest tests -m gpu -q --durations=12 > gpurun_out/r/gputests.log 2>&1; echo rc=$? >> gpurun_out/r/gputests.log
du -sh gpurun_out
tail -3 gpurun_out/r/gputests.log; tail -1 gpurun_out/r/smoke.log
for f in gpurun_out/r/*.json; do echo $f $(python -c "import json; d=json.load(open('$f')); print(round(d['ms_per_step'],2), d.get('roofline',{}) and round(d['roofline']['frac'],3))" 2>&1 | tail -1); done
