# GPU pass (session 5h): SM work granularity: batch 1/2/4, slice 16/32/64/128 (per-query C3),
# match parity with slice 16 (more, smaller groups) and the defaults
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/t
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/t/build.log 2>&1
for b in 1 2 4; do GAMMA_SM_BATCH=$b timeout 300 python tools/sm_queries.py 3 > gpurun_out/t/q_b$b.log 2>&1; done
for s in 16 32 128; do GAMMA_SM_SLICE=$s timeout 300 python tools/sm_queries.py 3 > gpurun_out/t/q_s$s.log 2>&1; done
GAMMA_SM_SLICE=16 timeout 900 python -m pytest tests/test_gpu_match.py -m gpu -q -x -k "rmat or er or hub or motif" > gpurun_out/t/match_s16.log 2>&1; echo rc=$? >> gpurun_out/t/match_s16.log
tail -2 gpurun_out/t/match_s16.log
