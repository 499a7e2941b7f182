#!/bin/bash
# Same-box A/B of in-tree library variants on C2 (and heavy): usage tools/ab_c2.sh TAG variant...
# ("-" = the default libgamma.so).  Prints ms/step and the bitmap class time.
TAG=$1; shift
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
for rep in 1 2; do
for v in "$@"; do
  if [ "$v" = "-" ]; then unset GAMMA_LIB_VARIANT; else export GAMMA_LIB_VARIANT=$v; fi
  timeout 300 python bench.py --no-cpu-baseline --steps 10 > gpurun_out/${TAG}_c2_${v}_$rep.json 2>/dev/null
  timeout 300 python bench.py --no-cpu-baseline --workload heavy --steps 5 > gpurun_out/${TAG}_heavy_${v}_$rep.json 2>/dev/null
done; done
unset GAMMA_LIB_VARIANT
python - <<PY
import json,glob
for f in sorted(glob.glob("gpurun_out/${TAG}_*.json")):
    try:
        d=json.load(open(f)); print(f, round(d["ms_per_step"],3), {k:round(v["ms"],2) for k,v in d["kernels"].items()}, list(d["config"]["results"].values())[:3])
    except Exception as e: print(f, "ERR", e)
PY
