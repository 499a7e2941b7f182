#!/bin/bash
# C3 A/B of library variants (build.py tag; "-" = default), 10-step batched bench lines
TAG=$1; shift
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
for rep in 1 2; do for v in "$@"; do
  if [ "$v" = "-" ]; then unset GAMMA_LIB_VARIANT; else export GAMMA_LIB_VARIANT=$v; fi
  python bench.py --workload c3 --no-cpu-baseline --steps 10 > gpurun_out/${TAG}_${v}_$rep.json 2>/dev/null
  python -c "
import json; d=json.load(open('gpurun_out/${TAG}_${v}_$rep.json')); print('$v', round(d['ms_per_step'],2), d['step_ms'], d.get('sm_retries_per_step'))"
done; done
