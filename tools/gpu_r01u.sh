# GPU pass (session 5i): per-consumer slice (16 for extension consumers, 64 for the count level)
# + batch 2: match parity suite, per-query C3 at defaults and with SLICE_EXT=32, bench c3 10 steps
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/u
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/u/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_match.py -m gpu -q -x > gpurun_out/u/match.log 2>&1; echo rc=$? >> gpurun_out/u/match.log
timeout 300 python tools/sm_queries.py 3 > gpurun_out/u/q_def.log 2>&1
GAMMA_SM_SLICE_EXT=32 timeout 300 python tools/sm_queries.py 3 > gpurun_out/u/q_e32.log 2>&1
GAMMA_SM_SLICE_EXT=8 timeout 300 python tools/sm_queries.py 3 > gpurun_out/u/q_e8.log 2>&1
timeout 300 python bench.py --workload c3 --no-cpu-baseline --steps 10 > gpurun_out/u/bench_c3.json 2> gpurun_out/u/bench_c3.err
tail -2 gpurun_out/u/match.log
for f in gpurun_out/u/*.json; do echo $f $(python -c "import json; d=json.load(open('$f')); print(round(d['ms_per_step'],2), d['step_ms'])" 2>&1 | tail -1); done
