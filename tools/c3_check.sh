#!/bin/bash
# C3 check on the GPU box: SM parity tests, two batched 10-step bench lines, one sequential
TAG=${1:-m}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_match.py -m gpu -q -x > gpurun_out/${TAG}_tests.log 2>&1; tail -2 gpurun_out/${TAG}_tests.log
for i in 1 2; do
  python bench.py --workload c3 --no-cpu-baseline --steps 10 > gpurun_out/${TAG}_c3_$i.json 2>/dev/null
  python -c "
import json; d=json.load(open('gpurun_out/${TAG}_c3_$i.json')); print(round(d['ms_per_step'],2), d['step_ms'], d.get('sm_retries_per_step'), {k:round(v['ms']/10,1) for k,v in d['kernels'].items()}, round(d['roofline']['frac'],3))"
done
python bench.py --workload c3 --no-cpu-baseline --steps 5 --sm-sequential > gpurun_out/${TAG}_c3_seq.json 2>/dev/null
python -c "
import json; d=json.load(open('gpurun_out/${TAG}_c3_seq.json')); print('seq', round(d['ms_per_step'],2), d['step_ms'])"
