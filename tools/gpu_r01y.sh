# GPU pass (session 5m): does the nvidia-smi sampler cause the C3 host stalls? 10-step c3 with
# and without it, alternating
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/y
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/y/build.log 2>&1
for i in 1 2; do
timeout 300 python bench.py --workload c3 --no-cpu-baseline --steps 10 > gpurun_out/y/c3_clk$i.json 2>/dev/null
timeout 300 python bench.py --workload c3 --no-cpu-baseline --steps 10 --no-clocks > gpurun_out/y/c3_noclk$i.json 2>/dev/null
done
for f in gpurun_out/y/*.json; do echo $f $(python -c "import json; d=json.load(open('$f')); print(round(d['ms_per_step'],2), d['step_ms'])" 2>&1 | tail -1); done
