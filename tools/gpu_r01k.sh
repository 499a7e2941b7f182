# GPU pass (session 4c): SM staging-size sweep on C3, team-kernel register cap probe on C2,
# SM parity with tiny staging caps (stresses the global-scratch / direct-write fallbacks)
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/tune
B="import sys; sys.path.insert(0,'paper_conf_icde_hu0o23_b200'); import build; build.build(force=True"
python -c "$B)" > gpurun_out/tune/build.log 2>&1
GAMMA_SM_LMCAP=64 GAMMA_SM_OUTCAP=64 timeout 900 python -m pytest tests/test_gpu_match.py -q -x > gpurun_out/tune/match_tinycaps.log 2>&1; echo rc=$? >> gpurun_out/tune/match_tinycaps.log
for v in "1024 512" "512 256" "256 256" "512 512" "2048 512" "256 128"; do
  set -- $v
  GAMMA_SM_LMCAP=$1 GAMMA_SM_OUTCAP=$2 timeout 300 python bench.py --workload c3 --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/tune/c3_$1_$2.json 2>/dev/null
done
timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/tune/c2_minb1.json 2>/dev/null
python -c "$B, extra=['-DGAMMA_BM_MINB=5'])" >> gpurun_out/tune/build.log 2>&1
timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/tune/c2_minb5.json 2>/dev/null
timeout 300 python bench.py --workload heavy --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/tune/heavy_minb5.json 2>/dev/null
python -c "$B)" >> gpurun_out/tune/build.log 2>&1
timeout 300 python bench.py --workload heavy --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/tune/heavy_minb1.json 2>/dev/null
tail -2 gpurun_out/tune/match_tinycaps.log
for f in gpurun_out/tune/*.json; do echo $f $(python -c "import json,sys; d=json.load(open('$f')); print(round(d['ms_per_step'],2), d['config']['results'] if 'c3' in '$f' else '')" 2>&1 | cut -c1-200); done
