"""Top SASS lines by warp-stall samples of an ncu report: python scripts/ncu_hot.py rep [n]"""
import csv, io, subprocess, sys
path = sys.argv[1]; n = int(sys.argv[2]) if len(sys.argv) > 2 else 25
out = subprocess.run(["ncu", "-i", path, "--page", "source", "--csv", "--print-source", "sass"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hdr = rows[1]
ci = {h: i for i, h in enumerate(hdr)}
data = rows[2:]
tot = sum(int(r[ci["Warp Stall Sampling (All Samples)"]] or 0) for r in data)
data.sort(key=lambda r: -int(r[ci["Warp Stall Sampling (All Samples)"]] or 0))
print("total samples", tot)
for r in data[:n]:
    s = int(r[ci["Warp Stall Sampling (All Samples)"]] or 0)
    print(f"{s:7d} {100*s/tot:5.1f}%  {r[ci['Address']][-5:]}  {r[ci['Source']].strip()[:90]}  exec={r[ci['Instructions Executed']]}")
