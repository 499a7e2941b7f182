#!/bin/bash
# Quick kCL loop on the GPU box: parity subset + C2/heavy bench lines, A/B against the
# list-streaming row build (GAMMA_KCL_NO_TABLES=1).  usage: tools/gpu_kcl_quick.sh TAG
TAG=${1:-q}
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_kclique.py -m gpu -q -x \
  -k "closed_forms or er_vs or c1_vs or per_root or complete_large or c2_full_size or heavy_full or paths_agree or parts_list or simulated_ranks or edge_cases" \
  > gpurun_out/${TAG}_tests.log 2>&1; tail -3 gpurun_out/${TAG}_tests.log
for v in 0 1; do
  GAMMA_KCL_NO_TABLES=$v timeout 300 python bench.py --no-cpu-baseline --steps 10 > gpurun_out/${TAG}_c2_t$v.json 2>/dev/null
  GAMMA_KCL_NO_TABLES=$v timeout 300 python bench.py --no-cpu-baseline --workload heavy --steps 5 > gpurun_out/${TAG}_heavy_t$v.json 2>/dev/null
done
python - <<PY
import json,glob
for f in sorted(glob.glob("gpurun_out/${TAG}_*.json")):
    try:
        d=json.load(open(f)); print(f, round(d["ms_per_step"],3), d["config"]["results"], d["kernels"].get("bitmap",{}).get("ms"))
    except Exception as e: print(f, "ERR", e)
PY
