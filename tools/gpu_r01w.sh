# GPU pass (session 5k): SM level tables kept across calls (no per-call allocator round trips):
# match + fpm + kclique parity, bench c3 10 steps x2, bench c2
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/w
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/w/smoke.log 2>&1; echo smoke rc=$? >> gpurun_out/w/smoke.log
timeout 1200 python -m pytest tests/test_gpu_match.py tests/test_gpu_fpm.py tests/test_gpu_kclique.py tests/test_gpu_dist.py -m gpu -q -x -k "not slow" > gpurun_out/w/tests.log 2>&1; echo rc=$? >> gpurun_out/w/tests.log
for i in 1 2; do timeout 300 python bench.py --workload c3 --no-cpu-baseline --steps 10 > gpurun_out/w/c3_$i.json 2>/dev/null; done
timeout 300 python bench.py > gpurun_out/w/c2.json 2>/dev/null
tail -2 gpurun_out/w/tests.log; tail -1 gpurun_out/w/smoke.log
for f in gpurun_out/w/*.json; do echo $f $(python -c "import json; d=json.load(open('$f')); print(round(d['ms_per_step'],2), d['step_ms'])" 2>&1 | tail -1); done
