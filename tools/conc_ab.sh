#!/bin/bash
# kCL: the concurrent warp-team launch vs one stream (GAMMA_KCL_SERIAL=1), C2 + heavy
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_kclique.py -m gpu -q -x \
  -k "closed_forms or er_vs or c1_vs or per_root or c2_full_size or heavy_full or paths_agree or parts_list" \
  > gpurun_out/conc_tests.log 2>&1; tail -2 gpurun_out/conc_tests.log
for rep in 1 2; do for v in 0 1; do
  GAMMA_KCL_SERIAL=$v python bench.py --no-cpu-baseline --steps 20 > gpurun_out/conc_c2_s${v}_$rep.json 2>/dev/null
  GAMMA_KCL_SERIAL=$v python bench.py --no-cpu-baseline --workload heavy --steps 5 > gpurun_out/conc_heavy_s${v}_$rep.json 2>/dev/null
done; done
python tools/show_bench.py gpurun_out/conc_*.json | cut -c1-140
