"""Summarise an ncu launch list (gpu__time_duration.sum per launch) of one
bench.py run: the last full inference step, kernel by kernel, in order."""
import csv, sys
rows = [r for r in csv.reader(open(sys.argv[1])) if len(r) > 10]
hdr = rows[0]
ik, iv = hdr.index("Kernel Name"), hdr.index("Metric Value")
ks = [(r[ik], float(r[iv].replace(",", ""))) for r in rows[1:] if r[hdr.index("Metric Name")] == "gpu__time_duration.sum"]
# steps start at the staging kernel
starts = [i for i, (k, _) in enumerate(ks) if k.startswith("stage")]
if len(starts) >= 2:
    seg = ks[starts[-2]:starts[-1]]
else:
    seg = ks[starts[-1]:] if starts else ks
unit = "ns" if max(v for _, v in seg) > 1000 else "us"
scale = 1e-3 if unit == "ns" else 1.0
tot = sum(v for _, v in seg) * scale
print("%s: %d launches, %.1f us total" % (sys.argv[2] if len(sys.argv) > 2 else "", len(seg), tot))
for k, v in seg:
    print("  %8.1f us  %s" % (v * scale, k[:70]))
