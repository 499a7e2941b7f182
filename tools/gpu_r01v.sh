# GPU pass (session 5j): C3 host-side step spread: default vs no cyclic GC vs native allocator
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/v
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/v/build.log 2>&1
for i in 1 2; do
timeout 300 python bench.py --workload c3 --no-cpu-baseline --steps 10 > gpurun_out/v/c3_def$i.json 2>/dev/null
GAMMA_BENCH_GC=0 timeout 300 python bench.py --workload c3 --no-cpu-baseline --steps 10 > gpurun_out/v/c3_nogc$i.json 2>/dev/null
GAMMA_ALLOC=native timeout 300 python bench.py --workload c3 --no-cpu-baseline --steps 10 > gpurun_out/v/c3_native$i.json 2>/dev/null
done
for f in gpurun_out/v/*.json; do echo $f $(python -c "import json; d=json.load(open('$f')); print(round(d['ms_per_step'],2), d['step_ms'])" 2>&1 | tail -1); done
