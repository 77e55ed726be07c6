#!/usr/bin/env python
"""Print the headline numbers and the top kernels of bench.py JSON lines (tooling)."""
import json
import sys

for f in sys.argv[1:]:
    try:
        for line in open(f):
            if not line.startswith("{"):
                continue
            d = json.loads(line)
            r = d.get("roofline", {})
            print(f, d.get("ms_per_step"), d.get("value"), r.get("kernel"), r.get("frac"), r.get("ms"))
            print("   ", {k: v for k, v in list(d.get("kernel_ms", {}).items())[:10]})
    except Exception as e:  # noqa: BLE001
        print(f, "error", e)
