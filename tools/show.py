#!/usr/bin/env python
"""Pretty-print bench JSON lines."""
import json
import sys
for ln in open(sys.argv[1]):
    try:
        d = json.loads(ln)
    except Exception:
        print("bad:", ln[:120]); continue
    c = d["config"]; r = d["roofline"]
    v = d.get("variant", "")
    print(f"V={v} {c['workload'][:24]:24s} T={c['T']:2d} tile={c['tile']} {d['value']:8.2f} GSt/s  "
          f"fused {r['achieved']:.2f} TF ({r['frac']:.3f}) mma {r['mma_tflops']:.2f} share={r['fused_share_of_step']:.3f}")
