#!/bin/bash
# ncu --set full of the dominant kernels of one timed step per workload (after 3 warm-up
# steps), summarised ON THE BOX (reports are too large to bring back): per-class JSON +
# markdown (tools/ncu_summary.py) and per-source-line tables (tools/ncu_lines.py) land in
# gpurun_out/profsum/; plus the C2 launch list (gpu__time_duration, the bench's command).
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/profsum
prof() {  # name regex skip count bench-args...
  local name=$1 rx=$2 skip=$3 cnt=$4; shift 4
  ncu --set full --clock-control none --import-source on -k regex:$rx --launch-skip $skip --launch-count $cnt \
    -o /tmp/prof_$name -f python bench.py "$@" --steps 1 --warmup 3 --no-cpu-baseline --no-clocks > gpurun_out/profsum/prof_$name.log 2>&1
  python tools/ncu_summary.py /tmp/prof_$name.ncu-rep gpurun_out/profsum r02b $name > gpurun_out/profsum/sum_$name.txt 2>&1
  for i in $(seq 0 $((cnt - 1))); do
    python tools/ncu_lines.py /tmp/prof_$name.ncu-rep --skip $i --top 40 > gpurun_out/profsum/lines_${name}_$i.txt 2>&1
  done
  rm -f /tmp/prof_$name.ncu-rep
}
prof c2 kcl_bitmap 9 3 --workload c2
prof heavy kcl_bitmap 6 2 --workload heavy
prof c3 sm_kernel 78 26 --workload c3
ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/profsum/launches_c2.csv \
  python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-clocks > /dev/null 2>&1
ls gpurun_out/profsum
