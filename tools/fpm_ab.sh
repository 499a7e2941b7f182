#!/bin/bash
# FPM: parity tests + C4 bench lines, default library vs variants (build.py tag)
TAG=$1; shift
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_fpm.py tests/test_gpu_dist.py -m gpu -q -x > gpurun_out/${TAG}_tests.log 2>&1; tail -2 gpurun_out/${TAG}_tests.log
for v in "$@"; do
  if [ "$v" = "-" ]; then unset GAMMA_LIB_VARIANT; else export GAMMA_LIB_VARIANT=$v; fi
  timeout 900 python bench.py --workload c4 --no-cpu-baseline --steps 3 > gpurun_out/${TAG}_c4_$v.json 2>/dev/null
done
unset GAMMA_LIB_VARIANT
python tools/show_bench.py gpurun_out/${TAG}_c4_*.json
python -c "
import json,glob
for f in sorted(glob.glob('gpurun_out/${TAG}_c4_*.json')):
    d=json.load(open(f)); print(f, d['config']['results'])"
