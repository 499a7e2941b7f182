#!/usr/bin/env python3
"""Summarise an ncu launch list (`ncu --metrics gpu__time_duration.sum --csv
--log-file X`) into per-kernel totals and shares (markdown).

    python tools/launch_summary.py gpurun_out/launches.csv profiles/launches_r01.md "<command>"
"""
import collections
import csv
import sys


def main():
    src, dst = sys.argv[1], sys.argv[2]
    cmd = sys.argv[3] if len(sys.argv) > 3 else ""
    rows = list(csv.reader(open(src)))
    hdr = None
    agg = collections.OrderedDict()
    n = 0
    for r in rows:
        if len(r) > 5 and r[0] == "ID":
            hdr = r
            continue
        if hdr is None or len(r) != len(hdr):
            continue
        d = dict(zip(hdr, r))
        if d.get("Metric Name") != "gpu__time_duration.sum":
            continue
        try:
            v = float(d["Metric Value"].replace(",", ""))
        except ValueError:
            continue
        unit = d.get("Metric Unit", "ns")
        scale = {"nsecond": 1e-6, "ns": 1e-6, "usecond": 1e-3, "us": 1e-3, "msecond": 1.0, "ms": 1.0}.get(unit, 1e-6)
        name = d["Kernel Name"].split("(")[0]
        a = agg.setdefault(name, [0, 0.0])
        a[0] += 1
        a[1] += v * scale
        n += 1
    tot = sum(v[1] for v in agg.values())
    lines = [f"ncu launch list ({n} launches, cold-cache serialised; compare shares, not absolutes)",
             f"command: `{cmd}`", "", "| kernel | launches | total ms | share |", "|---|---|---|---|"]
    for k, (c, ms) in sorted(agg.items(), key=lambda x: -x[1][1]):
        lines.append(f"| `{k[:90]}` | {c} | {ms:.3f} | {100 * ms / tot:.1f}% |")
    open(dst, "w").write("\n".join(lines) + "\n")
    print("\n".join(lines[:20]))


if __name__ == "__main__":
    main()
