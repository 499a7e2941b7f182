# GPU pass (session 4d): new defaults (team kernels min 5 CTAs/SM for k<=6, SM staging 512/512):
# full -m gpu suite (incl. the new full-size C3 parity), bench lines, MINB=6 probe, ncu of c2/c3
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/l/prof
B="import sys; sys.path.insert(0,'paper_conf_icde_hu0o23_b200'); import build; build.build(force=True"
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/l/smoke.log 2>&1; echo smoke rc=$? >> gpurun_out/l/smoke.log
timeout 1800 python -m pytest tests -m gpu -q --durations=12 > gpurun_out/l/gputests.log 2>&1; echo rc=$? >> gpurun_out/l/gputests.log
timeout 400 python bench.py > gpurun_out/l/bench_c2.json 2> gpurun_out/l/bench_c2.err
timeout 300 python bench.py --workload c1 > gpurun_out/l/bench_c1.json 2> gpurun_out/l/bench_c1.err
timeout 300 python bench.py --workload heavy --no-cpu-baseline > gpurun_out/l/bench_heavy.json 2> gpurun_out/l/bench_heavy.err
timeout 600 python bench.py --workload c3 --no-cpu-baseline > gpurun_out/l/bench_c3.json 2> gpurun_out/l/bench_c3.err
timeout 900 python bench.py --workload c4 --no-cpu-baseline --steps 3 --warmup 3 > gpurun_out/l/bench_c4.json 2> gpurun_out/l/bench_c4.err
timeout 900 python bench.py --workload c5 --steps 2 --warmup 3 > gpurun_out/l/bench_c5.json 2> gpurun_out/l/bench_c5.err
timeout 300 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/l/bench_ref.json 2> gpurun_out/l/bench_ref.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file /tmp/launches_c2.csv \
  python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-clocks > /dev/null 2>&1
python tools/launch_summary.py /tmp/launches_c2.csv gpurun_out/l/prof/launches_c2_r01.md "ncu --metrics gpu__time_duration.sum --clock-control none --csv python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-clocks"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file /tmp/launches_c3.csv \
  python bench.py --workload c3 --steps 1 --warmup 1 --no-cpu-baseline --no-clocks > /dev/null 2>&1
python tools/launch_summary.py /tmp/launches_c3.csv gpurun_out/l/prof/launches_c3_r01.md "ncu --metrics gpu__time_duration.sum --clock-control none --csv python bench.py --workload c3 --steps 1 --warmup 1 --no-cpu-baseline --no-clocks"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:kcl_bitmap -c 3 -o /tmp/ncu_c2 -f \
  python bench.py --steps 1 --warmup 0 --no-cpu-baseline --no-clocks > gpurun_out/l/ncu_c2.log 2>&1
python tools/ncu_summary.py /tmp/ncu_c2.ncu-rep gpurun_out/l/prof r01 c2 >> gpurun_out/l/ncu_c2.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:sm_kernel -s 6 -c 6 -o /tmp/ncu_c3 -f \
  python bench.py --workload c3 --steps 1 --warmup 0 --no-cpu-baseline --no-clocks > gpurun_out/l/ncu_c3.log 2>&1
python tools/ncu_summary.py /tmp/ncu_c3.ncu-rep gpurun_out/l/prof r01 c3 >> gpurun_out/l/ncu_c3.log 2>&1
python -c "$B, extra=['-DGAMMA_BM_MINB=6'])" > gpurun_out/l/build6.log 2>&1
timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/l/c2_minb6.json 2>/dev/null
timeout 300 python bench.py --workload heavy --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/l/heavy_minb6.json 2>/dev/null
python -c "$B)" >> gpurun_out/l/build6.log 2>&1
du -sh gpurun_out
tail -3 gpurun_out/l/gputests.log; tail -1 gpurun_out/l/smoke.log
for f in gpurun_out/l/*.json; do echo $f $(python -c "import json; d=json.load(open('$f')); print(round(d['ms_per_step'],2))" 2>&1 | tail -1); done
