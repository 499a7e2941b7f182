# GPU pass (session 5e): host-side variance of match calls: torch caching allocator vs the
# library's stream-ordered pool (GAMMA_ALLOC=native), per-rep wall + bench c3 10 steps each
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/q
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/q/build.log 2>&1
SMQ_ALL=1 timeout 300 python tools/sm_queries.py 5 > gpurun_out/q/q_torch.log 2>&1
SMQ_ALL=1 GAMMA_ALLOC=native timeout 300 python tools/sm_queries.py 5 > gpurun_out/q/q_native.log 2>&1
timeout 300 python bench.py --workload c3 --no-cpu-baseline --steps 10 > gpurun_out/q/bench_c3_torch.json 2> gpurun_out/q/bench_c3_torch.err
GAMMA_ALLOC=native timeout 300 python bench.py --workload c3 --no-cpu-baseline --steps 10 > gpurun_out/q/bench_c3_native.json 2> gpurun_out/q/bench_c3_native.err
GAMMA_ALLOC=native timeout 600 python -m pytest tests/test_gpu_fpm.py tests/test_gpu_match.py -m gpu -q -x -k "not slow" > gpurun_out/q/native_tests.log 2>&1; echo rc=$? >> gpurun_out/q/native_tests.log
for t in torch native; do echo "== $t"; grep "^  rep" gpurun_out/q/q_$t.log | awk '{print $2, $3}' | tr '\n' ' '; echo; done
tail -2 gpurun_out/q/native_tests.log
for f in gpurun_out/q/*.json; do echo $f $(python -c "import json; d=json.load(open('$f')); print(round(d['ms_per_step'],2), d['step_ms'])" 2>&1 | tail -1); done
