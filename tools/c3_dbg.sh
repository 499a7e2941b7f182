#!/bin/bash
# C3 host-side phase timing (GAMMA_DEBUG) next to the bench's step/host/kernel times
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
GAMMA_DEBUG=1 python bench.py --workload c3 --no-cpu-baseline --steps 10 $1 2> gpurun_out/dbg.err > gpurun_out/dbg.json
grep "sm batch" gpurun_out/dbg.err | tail -20 | cut -c1-40,100-200
python tools/show_bench.py gpurun_out/dbg.json
