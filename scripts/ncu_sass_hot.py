"""Top SASS lines by warp-stall samples of one kernel in an ncu report:
    python scripts/ncu_sass_hot.py rep.ncu-rep <kernel-regex> [n]"""
import csv, io, subprocess, sys
rep, kre = sys.argv[1], sys.argv[2]
n = int(sys.argv[3]) if len(sys.argv) > 3 else 25
out = subprocess.run(["ncu", "-i", rep, "-k", "regex:" + kre, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
blocks, cur = [], None
for r in rows:
    if r and r[0] == "Kernel Name":
        cur = {"name": r[1], "rows": []}; blocks.append(cur); continue
    if r and r[0] == "Address":
        cur["hdr"] = {h: i for i, h in enumerate(r)}; continue
    if cur is not None and "hdr" in cur and r:
        cur["rows"].append(r)
key = "Warp Stall Sampling (All Samples)"
for b in blocks[:1]:
    ci = b["hdr"]
    data = [r for r in b["rows"] if r[ci[key]].isdigit()]
    tot = sum(int(r[ci[key]]) for r in data)
    print(b["name"][:80], "samples", tot)
    for r in sorted(data, key=lambda r: -int(r[ci[key]]))[:n]:
        s = int(r[ci[key]])
        print(f"{s:7d} {100*s/max(tot,1):5.1f}%  {r[ci['Address']][-5:]}  {r[ci['Source']].strip()[:70]:70s} exec={r[ci['Instructions Executed']]}")
