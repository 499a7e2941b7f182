cd $GRAFT_REPO_ROOT
nvidia-smi --query-gpu=name,memory.total,clocks.sm --format=csv > gpurun_out/c5_smi.txt
timeout 1500 python tools/c5_probe.py --a 0.50 --samples 2.0e9 --a 0.55 --samples 2.0e9 --a 0.57 --samples 2.1e9 > gpurun_out/c5_probe.jsonl 2> gpurun_out/c5_probe.err
echo rc=$? >> gpurun_out/c5_probe.err
tail -5 gpurun_out/c5_probe.err; cat gpurun_out/c5_probe.jsonl
