"""Summarise ncu output for profiles/: a `--set full` report (.ncu-rep) or a launch-list CSV.

    python scripts/ncu_summary.py report gpurun_out/prof.ncu-rep
    python scripts/ncu_summary.py launches gpurun_out/launches.csv [--steps-skip N]
"""
import csv
import io
import subprocess
import sys
from collections import defaultdict

KEYS = [
    ("gpu__time_duration.sum", "dur"),
    ("launch__grid_size", "grid"),
    ("launch__registers_per_thread", "regs"),
    ("dram__bytes_read.sum", "dram_rd"),
    ("dram__bytes_write.sum", "dram_wr"),
    ("sm__ops_path_tensor_op_utchmma_src_bf16_dst_fp32_sparsity_off.avg.pct_of_peak_sustained_elapsed", "tc_bf16_%"),
    ("sm__pipe_tensor_cycles_active_realtime.avg.pct_of_peak_sustained_elapsed", "tensor_pipe_%"),
    ("TPC.TriageCompute.sm__pipe_tensor_cycles_active_realtime.avg.pct_of_peak_sustained_elapsed", "tensor_pipe_%"),
    ("lts__throughput.avg.pct_of_peak_sustained_elapsed", "L2_%"),
    ("dram__throughput.avg.pct_of_peak_sustained_elapsed", "dram_%"),
    ("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "dram_%"),
    ("sm__throughput.avg.pct_of_peak_sustained_elapsed", "sm_%"),
    ("lts__t_bytes.sum", "L2_bytes"),
]


def report(path):
    out = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units = rows[0], rows[1]
    col = {h: i for i, h in enumerate(hdr)}
    for r in rows[2:]:
        print(f"kernel: {r[col['Kernel Name']][:80]}")
        seen = set()
        for k, short in KEYS:
            if k in col and short not in seen:
                seen.add(short)
                print(f"  {short:14s} {r[col[k]]:>14s} {units[col[k]]}")


def launches(path, skip=0):
    rows = []
    with open(path) as f:
        lines = [l for l in f if l.startswith('"')]
    rd = csv.DictReader(io.StringIO("".join(lines)))
    for r in rd:
        if r.get("Metric Name") == "gpu__time_duration.sum":
            v = float(r["Metric Value"].replace(",", ""))
            unit = r.get("Metric Unit", "ns")
            scale = {"ns": 1e-3, "usecond": 1.0, "us": 1.0, "msecond": 1e3, "ms": 1e3, "nsecond": 1e-3}.get(unit, 1e-3)
            rows.append((int(r["ID"]), r["Kernel Name"], v * scale))
    rows.sort()
    tot = defaultdict(float)
    cnt = defaultdict(int)
    for _, name, us in rows[skip:]:
        k = name.split("(")[0].split("<")[0]
        tot[k] += us
        cnt[k] += 1
    allus = sum(tot.values())
    print(f"{len(rows) - skip} launches, {allus / 1e3:.3f} ms total (serialised, cold-cache)")
    for k, v in sorted(tot.items(), key=lambda kv: -kv[1]):
        print(f"  {k:40s} n={cnt[k]:5d}  {v / 1e3:9.3f} ms  {100 * v / allus:5.1f}%")


if __name__ == "__main__":
    if sys.argv[1] == "report":
        report(sys.argv[2])
    else:
        skip = int(sys.argv[sys.argv.index("--skip") + 1]) if "--skip" in sys.argv else 0
        launches(sys.argv[2], skip)
