"""Top SASS instructions by warp-stall samples from an ncu report (source page)."""
import csv, subprocess, sys
rep = sys.argv[1]
n = int(sys.argv[2]) if len(sys.argv) > 2 else 25
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(out.splitlines()))
hdr = rows[1]
ia, isrc, isamp = hdr.index("Address"), hdr.index("Source"), hdr.index("Warp Stall Sampling (All Samples)")
body = [r for r in rows[2:] if len(r) > isamp]
tot = sum(int(r[isamp] or 0) for r in body)
print("total samples", tot)
idx = {r[ia]: i for i, r in enumerate(body)}
for r in sorted(body, key=lambda r: -int(r[isamp] or 0))[:n]:
    i = idx[r[ia]]
    ctx = " | ".join(body[j][isrc].strip()[:40] for j in range(max(0, i - 2), i))
    print("%6s %5.1f%%  %-60s  <- %s" % (r[isamp], 100.0 * int(r[isamp]) / tot, r[isrc].strip()[:60], ctx))
