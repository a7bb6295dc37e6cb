#!/usr/bin/env python
"""Markdown rows of DESIGN §7 from bench JSON lines: python tools/r02_table.py file..."""
import json
import sys

for f in sys.argv[1:]:
    try:
        d = json.loads(open(f).read().strip().splitlines()[-1])
    except Exception as e:  # noqa: BLE001
        print(f"| {f} | unreadable: {e} |")
        continue
    r = d.get("roofline") or {}
    ph = r.get("phases") or {}
    n = d.get("steps", 1)
    per = ", ".join(f"{k} {v['ms'] * 1e3 / n:.1f}" for k, v in ph.items())
    e2e = (d.get("e2e") or {}).get("value")
    print(f"| {d['config']['workload']} | {d['value']} | {d['ms_per_step']} | {r.get('frac')} | "
          f"{r.get('traffic')} | {e2e} | {per} | {d.get('validated_roots')} |")
