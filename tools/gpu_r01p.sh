# GPU pass (session 5d): C3 step variance: per-rep wall vs kernel time and retries, bench c3 10 steps
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/p
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/p/build.log 2>&1
SMQ_ALL=1 timeout 300 python tools/sm_queries.py 5 > gpurun_out/p/q_all.log 2>&1
timeout 300 python bench.py --workload c3 --no-cpu-baseline --steps 10 > gpurun_out/p/bench_c3_10.json 2> gpurun_out/p/bench_c3_10.err
grep -v "^  rep" gpurun_out/p/q_all.log | cut -c1-80
for f in gpurun_out/p/*.json; do echo $f $(python -c "import json; d=json.load(open('$f')); print(round(d['ms_per_step'],2), d['step_ms'])" 2>&1 | tail -1); done
