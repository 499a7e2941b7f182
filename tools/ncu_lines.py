#!/usr/bin/env python3
"""Per-source-line breakdown of one kernel launch from an `ncu --set full
--import-source on` report: warp instructions executed, thread-instruction SIMT
efficiency and warp-stall samples per CUDA source line (needs -lineinfo).

    python tools/ncu_lines.py <report.ncu-rep> [--skip N] [--top 25] [--by inst|stall]
"""
import argparse
import csv
import io
import subprocess


def load(rep, skip):
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass",
                          "--launch-skip", str(skip), "--launch-count", "1"], capture_output=True, text=True).stdout
    rows, path, hdr = [], None, None
    for rec in csv.reader(io.StringIO(out)):
        if not rec:
            continue
        if rec[0] == "File Path":
            path = rec[1].split("/")[-1]
            continue
        if rec[0] == "Function Name":
            fn = rec[1]
            continue
        if rec[0] == "Line No":
            hdr = rec
            continue
        if hdr is None or rec[0] in ("", "..."):
            continue
        d = dict(zip(hdr[4:], rec[4:]))

        def num(k):
            try:
                return float(d.get(k, "0").replace(",", ""))
            except ValueError:
                return 0.0
        rows.append({"file": path, "line": int(rec[0]), "src": rec[1].strip(),
                     "inst": num("Instructions Executed"), "thr": num("Thread Instructions Executed"),
                     "stall": num("Warp Stall Sampling (All Samples)")})
    return fn, rows


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("rep")
    ap.add_argument("--skip", type=int, default=0)
    ap.add_argument("--top", type=int, default=25)
    ap.add_argument("--by", default="inst", choices=["inst", "stall"])
    a = ap.parse_args()
    fn, rows = load(a.rep, a.skip)
    ti = sum(r["inst"] for r in rows) or 1
    ts = sum(r["stall"] for r in rows) or 1
    print(f"{fn}\n  warp instructions {ti:.4g}, stall samples {ts:.4g}")
    print(f"  {'file:line':28s} {'inst%':>6s} {'stall%':>6s} {'thr/inst':>8s}  source")
    for r in sorted(rows, key=lambda r: -r[a.by])[:a.top]:
        eff = r["thr"] / r["inst"] if r["inst"] else 0
        print(f"  {r['file'] + ':' + str(r['line']):28s} {100 * r['inst'] / ti:6.2f} {100 * r['stall'] / ts:6.2f} "
              f"{eff:8.1f}  {r['src'][:90]}")


if __name__ == "__main__":
    main()
