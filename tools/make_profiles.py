"""Turn the raw ncu outputs of tools/prof_r01.sh (gpurun_out/<dir>/) into the
committed, per-round summaries under profiles/:

  profiles/<round>_launches_<net>_bf16.csv   one step's launch list (median over steps)
  profiles/<round>_full_<net>_bf16.csv       per-launch ncu --set full summary
  profiles/<round>_summary.md                shares of the step, dram traffic, tensor util
  profiles/ncu_summary.json                  dram bytes per conv launch (bench.py's roofline.traffic)

usage: python tools/make_profiles.py gpurun_out/r01b r01 [out_dir (default profiles/)]
"""
import csv
import json
import os
import statistics
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
BATCH = {"alexnet": 256, "vgg16": 64}
N_CONV = {"alexnet": 5, "vgg16": 13}   # conv layers come first; FC layers reuse the kernel


def short(name):
    name = name.replace("void ", "")
    return name.split("(")[0]


def read_launches(path):
    rows = []
    with open(path) as f:
        lines = [l for l in f if l.startswith('"')]
    for r in csv.DictReader(lines):
        if r.get("Metric Name") != "gpu__time_duration.sum":
            continue
        v = float(r["Metric Value"].replace(",", ""))
        unit = r["Metric Unit"]
        ns = v * {"ns": 1, "us": 1e3, "usecond": 1e3, "ms": 1e6, "msecond": 1e6}.get(unit, 1)
        rows.append((short(r["Kernel Name"]), r["Grid Size"], r["Block Size"], ns))
    return rows


def split_steps(rows):
    """Launches of one step are a fixed sequence beginning with the input
    staging kernel; return the steps of the modal length."""
    first = rows[0][0]
    steps, cur = [], []
    for r in rows:
        if r[0] == first and cur:
            steps.append(cur)
            cur = []
        cur.append(r)
    if cur:
        steps.append(cur)
    modal = statistics.mode(len(s) for s in steps)
    return [s for s in steps if len(s) == modal]


def launch_summary(path, out_csv):
    steps = split_steps(read_launches(path))
    n = len(steps[0])
    med = [statistics.median(s[i][3] for s in steps) for i in range(n)]
    total = sum(med)
    with open(out_csv, "w") as f:
        w = csv.writer(f)
        w.writerow(["pos", "kernel", "grid", "block", "median_ns", "share_of_step"])
        for i in range(n):
            k, g, b, _ = steps[0][i]
            w.writerow([i, k, g, b, round(med[i]), round(med[i] / total, 4)])
    by = {}
    for i in range(n):
        by[steps[0][i][0]] = by.get(steps[0][i][0], 0) + med[i]
    return dict(steps=len(steps), launches_per_step=n, step_ns=total,
                share={k: round(v / total, 4) for k, v in sorted(by.items(), key=lambda t: -t[1])})


METRICS = [("dur_ns", "gpu__time_duration.sum"), ("grid", "launch__grid_size"),
           ("block", "launch__block_size"), ("regs", "launch__registers_per_thread"),
           ("dram_read_B", "dram__bytes_read.sum"), ("dram_write_B", "dram__bytes_write.sum"),
           ("tensor_bf16_pct", "sm__ops_path_tensor_op_utchmma_src_bf16_dst_fp32_sparsity_off"
                               ".avg.pct_of_peak_sustained_elapsed"),
           ("dram_pct", "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed"),
           ("l2_pct", "lts__throughput.avg.pct_of_peak_sustained_elapsed"),
           ("l1_pct", "l1tex__throughput.avg.pct_of_peak_sustained_active"),
           ("sm_mhz", "sm__cycles_elapsed.avg.per_second")]


def full_summary(rep, out_csv):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"],
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(out.splitlines()))
    hdr, units = rows[0], rows[1]
    recs = []
    for r in rows[2:]:
        d = {"kernel": short(r[hdr.index("Kernel Name")])}
        for key, m in METRICS:
            if m not in hdr:
                d[key] = None
                continue
            raw = r[hdr.index(m)].replace(",", "")
            u = units[hdr.index(m)]
            try:
                v = float(raw)
            except ValueError:
                d[key] = raw
                continue
            scale = {"Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "KB": 1e3, "MB": 1e6, "GB": 1e9,
                     "usecond": 1e3, "us": 1e3, "msecond": 1e6, "ms": 1e6,
                     "Ghz": 1e3, "GHz": 1e3, "Mhz": 1, "MHz": 1, "hz": 1e-6, "Hz": 1e-6}
            if key == "sm_mhz":
                v *= scale.get(u, 1e-6) if u not in ("Mhz", "MHz") else 1
            else:
                v *= scale.get(u, 1)
            d[key] = v
        recs.append(d)
    with open(out_csv, "w") as f:
        w = csv.writer(f)
        w.writerow(["launch"] + list(recs[0].keys()))
        for i, d in enumerate(recs):
            w.writerow([i] + [(round(v, 3) if isinstance(v, float) else v) for v in d.values()])
    return recs


def main():
    src, rnd = sys.argv[1], sys.argv[2]
    prof = sys.argv[3] if len(sys.argv) > 3 else os.path.join(ROOT, "profiles")
    os.makedirs(prof, exist_ok=True)
    summ_path = os.path.join(prof, "ncu_summary.json")
    summary = json.load(open(summ_path)) if os.path.exists(summ_path) else {}
    md = ["# %s ncu summaries (B200, `--clock-control none`)" % rnd, "",
          "Generated by `tools/make_profiles.py %s %s` from the outputs of "
          "`tools/prof_r01.sh` (launch list = `ncu --metrics gpu__time_duration.sum` over "
          "`bench.py --steps 2 --warmup 3`; full = `ncu --set full -k regex:conv_tc_kernel`). "
          "ncu times are cold-cache and serialised: compare SHARES with bench.py's per_layer, "
          "not absolutes." % (src, rnd), ""]
    for net in ("alexnet", "vgg16"):
        lpath = os.path.join(src, "launches_%s_bf16.csv" % net)
        if os.path.exists(lpath):
            s = launch_summary(lpath, os.path.join(prof, "%s_launches_%s_bf16.csv" % (rnd, net)))
            md += ["## %s bf16, batch %d: launch list" % (net, BATCH[net]), "",
                   "%d steps parsed, %d launches per step, %.1f us per step (sum of serialised kernels)"
                   % (s["steps"], s["launches_per_step"], s["step_ns"] / 1e3), "",
                   "| kernel | share of step |", "|---|---|"]
            md += ["| %s | %.1f%% |" % (k, 100 * v) for k, v in s["share"].items()]
            md.append("")
        rep = os.path.join(src, "full_%s_bf16.ncu-rep" % net)
        if os.path.exists(rep):
            recs = full_summary(rep, os.path.join(prof, "%s_full_%s_bf16.csv" % (rnd, net)))
            conv = [d for d in recs if d["kernel"].startswith("conv_tc_kernel")][:N_CONV[net]]
            dram = [d["dram_read_B"] + d["dram_write_B"] for d in conv]
            key = "%s_bf16_b%d" % (net, BATCH[net])
            summary[key] = {
                "round": rnd,
                "conv_dram_bytes_per_launch": round(sum(dram) / len(dram)),
                "conv_launches": len(conv),
                "per_launch": [{"dur_us": round(d["dur_ns"] / 1e3, 2),
                                "dram_bytes": round(d["dram_read_B"] + d["dram_write_B"]),
                                "tensor_bf16_pct": d["tensor_bf16_pct"],
                                "l2_pct": d["l2_pct"]} for d in conv],
                "source": "ncu --set full, %s" % os.path.basename(rep)}
            md += ["## %s bf16, batch %d: conv layers (conv_tc_kernel), ncu --set full" % (net, BATCH[net]), "",
                   "| launch | us | grid | regs | DRAM read MB | DRAM write MB | tensor bf16 % | L2 % | DRAM % |",
                   "|---|---|---|---|---|---|---|---|---|"]
            for i, d in enumerate(conv):
                md.append("| %d | %.1f | %s | %s | %.1f | %.1f | %.1f | %.1f | %.1f |" % (
                    i, d["dur_ns"] / 1e3, d["grid"], d["regs"], d["dram_read_B"] / 1e6,
                    d["dram_write_B"] / 1e6, d["tensor_bf16_pct"] or 0, d["l2_pct"] or 0,
                    d["dram_pct"] or 0))
            md.append("")
    rep = os.path.join(src, "full_alexnet_other.ncu-rep")
    if os.path.exists(rep):
        recs = full_summary(rep, os.path.join(prof, "%s_full_alexnet_other_bf16.csv" % rnd))
        md += ["## alexnet bf16, batch 256: non-conv kernels, ncu --set full", "",
               "| kernel | us | grid | DRAM read MB | DRAM write MB | DRAM % | L2 % |",
               "|---|---|---|---|---|---|---|"]
        for d in recs:
            md.append("| %s | %.1f | %s | %.1f | %.1f | %.1f | %.1f |" % (
                d["kernel"], d["dur_ns"] / 1e3, d["grid"], d["dram_read_B"] / 1e6,
                d["dram_write_B"] / 1e6, d["dram_pct"] or 0, d["l2_pct"] or 0))
        md.append("")
    with open(summ_path, "w") as f:
        json.dump(summary, f, indent=1)
    with open(os.path.join(prof, "%s_summary.md" % rnd), "w") as f:
        f.write("\n".join(md) + "\n")


if __name__ == "__main__":
    main()
