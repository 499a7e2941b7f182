# GPU pass (session 5l): final validation of the round's HEAD: smoke, full -m gpu suite (incl.
# slow), bench c2 default line and c3
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/x
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/x/smoke.log 2>&1; echo smoke rc=$? >> gpurun_out/x/smoke.log
timeout 1800 python -m pytest tests -m gpu -q --durations=10 > gpurun_out/x/gputests.log 2>&1; echo rc=$? >> gpurun_out/x/gputests.log
timeout 400 python bench.py > gpurun_out/x/bench_c2.json 2> gpurun_out/x/bench_c2.err
timeout 300 python bench.py --workload c3 --no-cpu-baseline > gpurun_out/x/bench_c3.json 2> gpurun_out/x/bench_c3.err
tail -3 gpurun_out/x/gputests.log; tail -1 gpurun_out/x/smoke.log
for f in gpurun_out/x/*.json; do echo $f $(python -c "import json; d=json.load(open('$f')); print(round(d['ms_per_step'],2), d['step_ms'])" 2>&1 | tail -1); done
