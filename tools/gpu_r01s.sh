# GPU pass (session 5g): staged-candidate light filter (no label/degree gathers for L_m
# entries): match parity suite, per-query C3, work-queue batch sweep 4/8/16, bench c3
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/s
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/s/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_match.py -m gpu -q -x > gpurun_out/s/match.log 2>&1; echo rc=$? >> gpurun_out/s/match.log
for b in 4 8 16; do
  GAMMA_SM_BATCH=$b timeout 300 python tools/sm_queries.py 3 > gpurun_out/s/q_b$b.log 2>&1
done
timeout 300 python bench.py --workload c3 --no-cpu-baseline --steps 10 > gpurun_out/s/bench_c3.json 2> gpurun_out/s/bench_c3.err
tail -2 gpurun_out/s/match.log
for f in gpurun_out/s/*.json; do echo $f $(python -c "import json; d=json.load(open('$f')); print(round(d['ms_per_step'],2), d['step_ms'])" 2>&1 | tail -1); done
