# GPU pass (session 5): re-validate HEAD after the container restore: smoke, full -m gpu suite
# (incl. motif counting), bench c2 default line
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/m
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/m/smi.txt
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/m/smoke.log 2>&1; echo smoke rc=$? >> gpurun_out/m/smoke.log
timeout 1800 python -m pytest tests -m gpu -q --durations=15 > gpurun_out/m/gputests.log 2>&1; echo rc=$? >> gpurun_out/m/gputests.log
timeout 400 python bench.py > gpurun_out/m/bench_c2.json 2> gpurun_out/m/bench_c2.err
timeout 300 python bench.py --workload c3 --no-cpu-baseline > gpurun_out/m/bench_c3.json 2> gpurun_out/m/bench_c3.err
tail -3 gpurun_out/m/gputests.log; tail -1 gpurun_out/m/smoke.log
for f in gpurun_out/m/*.json; do echo $f $(python -c "import json; d=json.load(open('$f')); print(round(d['ms_per_step'],2))" 2>&1 | tail -1); done
