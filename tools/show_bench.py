#!/usr/bin/env python3
"""Print the timing fields of bench.py JSON lines: tools/show_bench.py file.json..."""
import json
import sys

for f in sys.argv[1:]:
    try:
        d = json.load(open(f))
    except (OSError, ValueError) as e:
        print(f, "ERR", e)
        continue
    print(f, round(d["ms_per_step"], 2), "steps", d.get("step_ms"), "kernels", d.get("step_kernel_ms"), "host", d.get("step_host_ms"),
          "retries", d.get("sm_retries_per_step"), "frac", round((d.get("roofline") or {}).get("frac") or 0, 3))
