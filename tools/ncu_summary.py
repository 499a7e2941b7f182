#!/usr/bin/env python3
"""Summarise an `ncu --set full` report into profiles/ncu_full_<class>.json (one file
per kernel class, averaged over the captured launches) plus a markdown table.

    python tools/ncu_summary.py gpurun_out/prof.ncu-rep profiles/ <round-tag> [<workload>]

With a workload name the files are profiles/ncu_<workload>_<class>.json (read by
bench.py's roofline "traffic" for that workload) and ncu_<workload>_<tag>.md.

Kernel classes follow the library's stats names: kcl_kernel<0,..> extend,
<1,..> count, <2,..> fused, kcl_bitmap_kernel bitmap, sm_kernel sm_extend,
fpm_enum_kernel fpm.
"""
import csv
import io
import json
import os
import re
import subprocess
import sys

METRICS = {
    "duration_ms": ("gpu__time_duration.sum", 1e-6),          # ns -> ms (unit checked below)
    "dram_read": ("dram__bytes_read.sum", 1.0),
    "dram_write": ("dram__bytes_write.sum", 1.0),
    "l2_hit_pct": ("lts__t_sector_hit_rate.pct", 1.0),
    "l1_hit_pct": ("l1tex__t_sector_hit_rate.pct", 1.0),
    "warps_active_pct": ("sm__warps_active.avg.pct_of_peak_sustained_active", 1.0),
    "sm_throughput_pct": ("sm__throughput.avg.pct_of_peak_sustained_elapsed", 1.0),
    "dram_throughput_pct": ("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", 1.0),
    "issue_active_pct": ("sm__inst_issued.avg.pct_of_peak_sustained_active", 1.0),
    "threads_per_warp_inst": ("smsp__thread_inst_executed_per_inst_executed.ratio", 1.0),
    "inst_executed": ("smsp__inst_executed.sum", 1.0),
    "registers": ("launch__registers_per_thread", 1.0),
    "grid": ("launch__grid_size", 1.0),
}
UNIT_SCALE = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "KB": 1e3, "MB": 1e6, "GB": 1e9,
              "nsecond": 1e-6, "usecond": 1e-3, "msecond": 1.0, "second": 1e3, "ns": 1e-6, "us": 1e-3,
              "ms": 1.0, "s": 1e3}


def kclass(name: str) -> str:
    if "kcl_bitmap_parts_kernel" in name:
        return "bitmap_parts"
    if "kcl_bitmap_kernel" in name:
        return "bitmap"
    m = re.search(r"kcl_kernel<(\d)", name)
    if m:
        return {"0": "extend", "1": "count", "2": "fused"}[m.group(1)]
    if "sm_kernel" in name:
        return "sm_extend"
    if "fpm_enum_kernel" in name:
        return "fpm"
    if "fpm_support" in name:
        return "fpm_support"
    return "other"


def main():
    rep, outdir, tag = sys.argv[1], sys.argv[2], sys.argv[3] if len(sys.argv) > 3 else "r01"
    prefix = f"ncu_{sys.argv[4]}_" if len(sys.argv) > 4 else "ncu_full_"
    raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    hdr, units = rows[0], rows[1]
    idx = {h: i for i, h in enumerate(hdr)}
    per = {}
    for r in rows[2:]:
        name = r[idx["Kernel Name"]]
        rec = {"kernel": name}
        for key, (metric, _) in METRICS.items():
            if metric not in idx:
                continue
            v = r[idx[metric]].replace(",", "")
            try:
                x = float(v)
            except ValueError:
                continue
            u = units[idx[metric]]
            if key == "duration_ms":
                x *= UNIT_SCALE.get(u, 1e-6)
            elif key in ("dram_read", "dram_write"):
                x *= UNIT_SCALE.get(u, 1)
            rec[key] = x
        per.setdefault(kclass(name), []).append(rec)
    os.makedirs(outdir, exist_ok=True)
    lines = [f"| class | launches | ms/launch | DRAM bytes/launch | L2 hit % | warps active % | issue active % | "
             f"SM thru % | DRAM thru % | regs |", "|---|---|---|---|---|---|---|---|---|---|"]
    for c, recs in sorted(per.items()):
        def avg(k):
            xs = [r[k] for r in recs if k in r]
            return sum(xs) / len(xs) if xs else None
        dram = (avg("dram_read") or 0) + (avg("dram_write") or 0)
        summary = {"class": c, "tag": tag, "launches_captured": len(recs), "ms_per_launch": avg("duration_ms"),
                   "dram_bytes_per_launch": dram, "l2_hit_pct": avg("l2_hit_pct"), "l1_hit_pct": avg("l1_hit_pct"),
                   "warps_active_pct": avg("warps_active_pct"), "issue_active_pct": avg("issue_active_pct"),
                   "sm_throughput_pct": avg("sm_throughput_pct"), "dram_throughput_pct": avg("dram_throughput_pct"),
                   "inst_executed_per_launch": avg("inst_executed"), "registers": avg("registers"),
                   "source": os.path.basename(rep), "launches": recs}
        summary["threads_per_warp_inst"] = avg("threads_per_warp_inst")
        with open(os.path.join(outdir, f"{prefix}{c}.json"), "w") as f:
            json.dump(summary, f, indent=1)
        fmt = lambda x, p=1: "-" if x is None else f"{x:.{p}f}"   # noqa: E731
        lines.append(f"| {c} | {len(recs)} | {fmt(avg('duration_ms'), 3)} | {dram:.3e} | {fmt(avg('l2_hit_pct'))} | "
                     f"{fmt(avg('warps_active_pct'))} | {fmt(avg('issue_active_pct'))} | "
                     f"{fmt(avg('sm_throughput_pct'))} | {fmt(avg('dram_throughput_pct'))} | {fmt(avg('registers'), 0)} |")
    with open(os.path.join(outdir, f"{prefix}{tag}.md"), "w") as f:
        f.write(f"ncu --set full summary of {os.path.basename(rep)} ({tag})\n\n" + "\n".join(lines) + "\n")
    print("\n".join(lines))


if __name__ == "__main__":
    main()
