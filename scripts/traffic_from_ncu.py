"""profiles/traffic_<cfg>.json from an ncu launch list with DRAM bytes of one bench step:
    ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --csv --log-file L.csv \\
        python bench.py --config C5 --steps 1 --warmup 3 --no-cpu-baseline
    python scripts/traffic_from_ncu.py L.csv C5 > profiles/traffic_C5.json
The timed step is the 4th (3 warm-up steps; a step starts with the input split launch and has two
split launches).  Conv family = conv_tc_kernel + wgrad_* launches (the tensor-core GEMMs); the
algorithmic bytes per conv pass follow SURVEY 8(d): (N*Cin*H*W + N*Cout*Ho*Wo)*2 + weights."""
import csv, io, json, sys
sys.path.insert(0, ".")
import synth

path, cfg = sys.argv[1], sys.argv[2] if len(sys.argv) > 2 else "C5"
rows = [l for l in open(path) if not l.startswith("==")]
by = {}
for x in csv.DictReader(io.StringIO("".join(rows))):
    d = by.setdefault(int(x["ID"]), {"k": x["Kernel Name"]})
    d[x["Metric Name"]] = float(x["Metric Value"].replace(",", ""))
L = [by[k] for k in sorted(by)]
starts = [i for i, x in enumerate(L) if "split_kernel" in x["k"]][::2]
s0, s1 = starts[3], starts[4]
step = L[s0:s1]
conv = [x for x in step if "conv_tc_kernel" in x["k"] or "wgrad_" in x["k"]]
dram = sum(x["dram__bytes_read.sum"] + x["dram__bytes_write.sum"] for x in conv)
allb = sum(x["dram__bytes_read.sum"] + x["dram__bytes_write.sum"] for x in step)
c = synth.vgg_config(cfg)
N, h = c["N"], c["H"]
alg, passes, first = 0.0, 0, True
for l in c["layers"] + c["tail"]:
    ho = (h + l["ph_b"] + l["ph_e"] - l["kh"]) // l["sh"] + 1
    if l["op"] == "conv":
        io_b = (N * l["cin"] * h * h + N * l["cout"] * ho * ho) * 2
        wb = l["cout"] * l["cin"] * l["kh"] * l["kw"]
        alg += io_b + 2 * wb                     # fwd
        alg += io_b + 4 * wb                     # wgrad (fp32 dW)
        passes += 2
        if not first:
            alg += io_b + 2 * wb                 # dgrad
            passes += 1
        first = False
    h = ho
out = {"config": cfg, "source": path.split("/")[-1],
       "conv_launches_in_step": len(conv), "conv_passes_in_step": passes,
       "conv_bytes_per_launch": round(dram / len(conv)),
       "conv_dram_bytes_per_step": round(dram), "conv_algorithmic_bytes_per_step": round(alg),
       "conv_dram_over_algorithmic": round(dram / alg, 3),
       "step_dram_bytes": round(allb),
       "note": "dram = dram__bytes_read.sum + dram__bytes_write.sum of the conv_tc / wgrad_* launches of one warm C5 step "
               "(ncu, --clock-control none, serialised); algorithmic = SURVEY 8(d) bytes of fwd+dgrad+wgrad of every conv"}
print(json.dumps(out, indent=1))
