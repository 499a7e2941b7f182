#!/bin/bash
# C3 knob sweep in the batched (default) bench mode: one bench line per setting.
# usage: tools/sm_sweep.sh TAG "ENV=.. ENV=.." ...
TAG=$1; shift
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
i=0
for cfg in "$@"; do
  i=$((i+1))
  env $cfg timeout 400 python bench.py --workload c3 --no-cpu-baseline --steps 5 > gpurun_out/${TAG}_$i.json 2>/dev/null
  python -c "
import json
d=json.load(open('gpurun_out/${TAG}_$i.json')); print('$cfg', round(d['ms_per_step'],2), d['step_ms'], {k:round(v['ms']/5,1) for k,v in d['kernels'].items()})
" 2>&1 | tail -1
done
