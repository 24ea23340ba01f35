"""Markdown table of committed bench lines (default profiles/r2_bench_*.json) for DESIGN.md §11.
    python scripts/summarize_round.py [glob]"""
import glob
import json
import os
import sys

pat = sys.argv[1] if len(sys.argv) > 1 else "profiles/r2_bench_*.json"
rows = []
for f in sorted(glob.glob(pat)):
    try:
        d = json.loads([l for l in open(f) if l.startswith("{")][-1])
    except Exception:
        continue
    if "unavailable" in d:
        continue
    rf = d.get("roofline") or {}
    hb = d.get("hbm_ops") or {}
    mem = d.get("memory") or {}
    rows.append((os.path.basename(f), d.get("config", {}).get("workload", "")[:60], d.get("dtype"), d.get("value"),
                 d.get("ms_per_step"), (d.get("e2e") or {}).get("value"), rf.get("achieved"), rf.get("frac"),
                 hb.get("achieved_gbs"), mem.get("peak_allocated_gb"), (d.get("clocks") or {}).get("sm_mhz")))
print("| file | workload | dtype | img/s | ms/step | e2e img/s | conv TFLOP/s | frac | pool/split/merge GB/s | peak GB | SM MHz |")
print("|---|---|---|---|---|---|---|---|---|---|---|")
for r in rows:
    print("| " + " | ".join("" if v is None else (f"{v:.4g}" if isinstance(v, float) else str(v)) for v in r) + " |")
