# GPU pass (session 5b): SM last-level long-child probe: parity (match suite incl. the
# ratio sweep test), per-query C3 timing at ratios 0 (off) / 4 / 8 / 16 / 32, bench c3
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/n
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/n/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_match.py -m gpu -q -x > gpurun_out/n/match.log 2>&1; echo rc=$? >> gpurun_out/n/match.log
for r in 0 8 4 16 32; do
  GAMMA_SM_LONGRATIO=$r timeout 300 python tools/sm_queries.py 2 > gpurun_out/n/q_$r.log 2>&1
done
timeout 300 python bench.py --workload c3 --no-cpu-baseline > gpurun_out/n/bench_c3.json 2> gpurun_out/n/bench_c3.err
GAMMA_SM_LONGRATIO=0 timeout 300 python bench.py --workload c3 --no-cpu-baseline > gpurun_out/n/bench_c3_off.json 2> gpurun_out/n/bench_c3_off.err
tail -2 gpurun_out/n/match.log
for r in 0 8 4 16 32; do echo "== ratio $r"; cut -c1-60 gpurun_out/n/q_$r.log; done
for f in gpurun_out/n/*.json; do echo $f $(python -c "import json; d=json.load(open('$f')); print(round(d['ms_per_step'],2), d['step_ms'])" 2>&1 | tail -1); done
