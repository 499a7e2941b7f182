#!/bin/bash
# Quick kCL loop on the GPU box: parity subset + C2/heavy bench lines + the per-band
# launch list of C2.  usage: tools/gpu_kcl_quick.sh TAG
TAG=${1:-q}
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_kclique.py -m gpu -q -x \
  -k "closed_forms or er_vs or c1_vs or per_root or complete_large or c2_full_size or heavy_full or paths_agree or parts_list or simulated_ranks or edge_cases" \
  > gpurun_out/${TAG}_tests.log 2>&1; tail -3 gpurun_out/${TAG}_tests.log
timeout 300 python bench.py --no-cpu-baseline --steps 10 > gpurun_out/${TAG}_c2.json 2>/dev/null
timeout 300 python bench.py --no-cpu-baseline --workload heavy --steps 5 > gpurun_out/${TAG}_heavy.json 2>/dev/null
GAMMA_KCL_BANDS=1 ncu --metrics gpu__time_duration.sum --clock-control none -c 200 --csv \
  --log-file gpurun_out/${TAG}_bands.csv python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-clocks > /dev/null 2>&1
python - <<PY
import json,glob,csv
for f in sorted(glob.glob("gpurun_out/${TAG}_*.json")):
    try:
        d=json.load(open(f)); print(f, round(d["ms_per_step"],3), d["config"]["results"], {k:round(v["ms"],2) for k,v in d["kernels"].items()})
    except Exception as e: print(f, "ERR", e)
rows=list(csv.reader(open("gpurun_out/${TAG}_bands.csv"))); hdr=None; out=[]
for r in rows:
    if r and r[0]=="ID": hdr=r; continue
    if hdr and len(r)==len(hdr):
        d=dict(zip(hdr,r))
        if "kcl" in d["Kernel Name"]: out.append(d["Metric Value"])
print("bands (CTA, 65-128, 33-64, 17-32, 9-16, 0-8, parts) ns:", out[-7:])
PY
# optional A/B variant library (build.py tag): GAMMA_LIB_VARIANT=$2
if [ -n "$2" ]; then
  GAMMA_LIB_VARIANT=$2 timeout 300 python bench.py --no-cpu-baseline --steps 10 > gpurun_out/${TAG}_c2_$2.json 2>/dev/null
  GAMMA_LIB_VARIANT=$2 timeout 300 python bench.py --no-cpu-baseline --workload heavy --steps 5 > gpurun_out/${TAG}_heavy_$2.json 2>/dev/null
  python -c "
import json
for f in ['gpurun_out/${TAG}_c2_$2.json','gpurun_out/${TAG}_heavy_$2.json']:
    d=json.load(open(f)); print(f, round(d['ms_per_step'],3), {k:round(v['ms'],2) for k,v in d['kernels'].items()})
"
fi
