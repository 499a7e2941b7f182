#!/bin/bash
# C3 step spread with and without the nvidia-smi clock sampler (diagnostic)
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
for rep in 1 2; do
  python bench.py --workload c3 --no-cpu-baseline --steps 10 > gpurun_out/al_c_$rep.json 2>/dev/null
  python bench.py --workload c3 --no-cpu-baseline --steps 10 --no-clocks > gpurun_out/al_n_$rep.json 2>/dev/null
done
python tools/show_bench.py gpurun_out/al_*.json
