"""Markdown table of the committed bench lines (profiles/r1_bench_*.json) for DESIGN.md §11."""
import glob, json, os, sys

rows = []
for f in sorted(glob.glob("profiles/r1_bench_*.json")):
    try:
        d = json.loads(open(f).read().strip().splitlines()[-1])
    except Exception:
        continue
    rf = d.get("roofline") or {}
    hb = d.get("hbm_ops") or {}
    mem = d.get("memory") or {}
    rows.append((os.path.basename(f), d.get("config", {}).get("workload", "")[:110], d.get("value"), d.get("ms_per_step"),
                 (d.get("e2e") or {}).get("value"), rf.get("achieved"), rf.get("frac"), hb.get("achieved_gbs"),
                 mem.get("peak_allocated_gb"), (d.get("clocks") or {}).get("sm_mhz")))
print("| file | workload | img/s | ms/step | e2e img/s | conv TFLOP/s | frac of peak | pool/split/merge GB/s | peak GB | SM MHz |")
print("|---|---|---|---|---|---|---|---|---|---|")
for r in rows:
    print("| " + " | ".join("" if v is None else (f"{v:.4g}" if isinstance(v, float) else str(v)) for v in r) + " |")
