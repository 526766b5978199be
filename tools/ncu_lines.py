"""Per-source-line stall summary of the kernels in an .ncu-rep (read here, not
on the GPU box):  python tools/ncu_lines.py report.ncu-rep [top] [function-substring]
Aggregates the SASS rows under each CUDA source line (--print-source cuda,sass)."""
import csv, io, subprocess, sys
rep = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 25
want = sys.argv[3] if len(sys.argv) > 3 else None
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
agg, src, cur, fname = {}, {}, None, ""
hdr = None
keep = True
for r in csv.reader(io.StringIO(out)):
    if not r:
        continue
    if r[0] == "Function Name":
        keep = want is None or want in r[1]
        continue
    if not keep:
        continue
    if r[0] == "File Path":
        fname = r[1].split("/")[-1]
        continue
    if r[0] == "Line No":
        hdr = r
        ist, iex = r.index("Warp Stall Sampling (All Samples)"), r.index("Instructions Executed")
        continue
    if hdr is None or len(r) <= ist:
        continue
    if r[0]:
        cur = (fname, int(r[0]))
        src[cur] = r[1]
        continue
    try:
        s, e = float(r[ist] or 0), float(r[iex] or 0)
    except ValueError:
        continue
    a = agg.setdefault(cur, [0.0, 0.0])
    a[0] += s
    a[1] += e
tot = sum(v[0] for v in agg.values()) or 1
print("stall samples", int(tot))
for k, v in sorted(agg.items(), key=lambda kv: -kv[1][0])[:top]:
    print("%5.1f%% ex=%-9d %s:%d  %s" % (100 * v[0] / tot, v[1], k[0], k[1], src[k].strip()[:90]))
