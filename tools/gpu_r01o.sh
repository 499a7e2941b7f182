# GPU pass (session 5c): long-child probe default ratio 4: match suite, per-query C3 at
# ratios 1 / 2 / 3 / 4, bench c3 with and without the nvidia-smi clock sampler (step variance)
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/o
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/o/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_match.py -m gpu -q -x > gpurun_out/o/match.log 2>&1; echo rc=$? >> gpurun_out/o/match.log
for r in 1 2 3 4; do
  GAMMA_SM_LONGRATIO=$r timeout 300 python tools/sm_queries.py 2 > gpurun_out/o/q_$r.log 2>&1
done
timeout 300 python bench.py --workload c3 --no-cpu-baseline > gpurun_out/o/bench_c3.json 2> gpurun_out/o/bench_c3.err
timeout 300 python bench.py --workload c3 --no-cpu-baseline --no-clocks > gpurun_out/o/bench_c3_noclk.json 2> gpurun_out/o/bench_c3_noclk.err
timeout 300 python bench.py --workload c3 --no-cpu-baseline --steps 10 > gpurun_out/o/bench_c3_10.json 2> gpurun_out/o/bench_c3_10.err
tail -2 gpurun_out/o/match.log
for f in gpurun_out/o/*.json; do echo $f $(python -c "import json; d=json.load(open('$f')); print(round(d['ms_per_step'],2), d['step_ms'])" 2>&1 | tail -1); done
