#!/usr/bin/env python
"""One row per bench JSON line: throughput, step time, whole-step and scan roofline fractions, clocks."""
import json
import sys

for line in open(sys.argv[1]):
    try:
        d = json.loads(line)
    except Exception:
        continue
    r = d["roofline"]
    c = d.get("clocks") or {}
    print(f'{d["config"]["workload"][:58]:58s} {d["value"]:.3e} t/s  ms={d["ms_per_step"]:7.2f}  '
          f'step={r.get("step_frac") or 0:.3f} scan={r["frac"] or 0:.3f} ({r["kernel"]}/{r["window_kernels"]}) '
          f'clk={c.get("sm_mhz")}/{c.get("samples")} {",".join(c.get("reasons") or [])}')
