"""Turn a round's raw ncu outputs (gpurun_out/) into the committed summaries
under profiles/ (see tools/gpu_prof_r02.sh for the commands that made them):

  <round>_launches_<tag>.csv   one inference step, kernel by kernel: median
                               gpu__time_duration over the complete steps of the
                               launch list (ncu --clock-control none; cold-cache,
                               serialised launches -- shares, not absolutes)
  <round>_ncu_full_<tag>.csv   per launch of the --set full capture: duration,
                               DRAM bytes, tensor-pipe and DRAM utilisation
  ncu_summary.json             DRAM bytes per conv launch (bench.py roofline.traffic)

usage: python tools/summarize_profiles.py r02
"""
import csv
import json
import os
import statistics
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
RND = sys.argv[1] if len(sys.argv) > 1 else "r02"
OUT = os.path.join(ROOT, "profiles")
RAW = os.path.join(ROOT, "gpurun_out")


def short(name):
    return name.replace("void ", "").split("(")[0]


def read_launches(path):
    rows = []
    with open(path) as f:
        lines = [l for l in f if l.startswith('"')]
    for r in csv.DictReader(lines):
        if r.get("Metric Name") != "gpu__time_duration.sum":
            continue
        v = float(r["Metric Value"].replace(",", ""))
        scale = {"ns": 1e-3, "nsecond": 1e-3, "us": 1.0, "usecond": 1.0, "ms": 1e3}.get(r["Metric Unit"], 1e-3)
        rows.append((short(r["Kernel Name"]), v * scale))
    return rows


def one_step(rows, first="stage"):
    starts = [i for i, (k, _) in enumerate(rows) if k.startswith(first)]
    steps = [rows[a:b] for a, b in zip(starts, starts[1:])]
    n = max(len(s) for s in steps)
    steps = [s for s in steps if len(s) == n]
    return [(steps[0][j][0], statistics.median(s[j][1] for s in steps)) for j in range(n)], len(steps)


summary = {}
for tag in ("alexnet_b256", "alexnet_b1", "vgg16_b64"):
    src = os.path.join(RAW, "launches_%s_%s.csv" % (tag, RND))
    if not os.path.exists(src):
        continue
    step, nsteps = one_step(read_launches(src))
    tot = sum(v for _, v in step)
    with open(os.path.join(OUT, "%s_launches_%s.csv" % (RND, tag)), "w") as f:
        f.write("kernel,us_median,share_of_step\n")
        for k, v in step:
            f.write("\"%s\",%.2f,%.4f\n" % (k, v, v / tot))
    summary[tag] = {"steps": nsteps, "launches_per_step": len(step), "sum_us": round(tot, 1),
                    "kernels": [[k, round(v, 2)] for k, v in step]}

full = os.path.join(RAW, "full_alexnet_b256_%s.ncu-rep" % RND)
if os.path.exists(full):
    raw = subprocess.run(["ncu", "-i", full, "--page", "raw", "--csv"], capture_output=True,
                         text=True).stdout.splitlines()
    rows = list(csv.reader(raw))
    h = rows[0]
    keys = ["Kernel Name", "Grid Size", "gpu__time_duration.sum", "dram__bytes_read.sum",
            "dram__bytes_write.sum", "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active",
            "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "launch__registers_per_thread"]
    idx = [h.index(k) for k in keys]
    units = [rows[1][i] for i in idx]
    out = []
    for r in rows[2:]:
        d = {k: r[i] for k, i in zip(keys, idx)}
        mb = lambda x: float(x) * (1e6 if "Mbyte" in units[3] else 1e9 if "Gbyte" in units[3] else 1e3)
        out.append({"kernel": short(d["Kernel Name"]), "grid": d["Grid Size"],
                    "dur_us": float(d["gpu__time_duration.sum"]),
                    "dram_bytes": int(mb(d["dram__bytes_read.sum"]) + mb(d["dram__bytes_write.sum"])),
                    "tensor_pct": float(d["sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active"]),
                    "dram_pct": float(d["gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed"]),
                    "regs": int(float(d["launch__registers_per_thread"]))})
    with open(os.path.join(OUT, "%s_ncu_full_alexnet_b256.csv" % RND), "w") as f:
        f.write("kernel,grid,dur_us,dram_bytes,tensor_pipe_pct,dram_pct,regs\n")
        for d in out:
            f.write("\"%s\",\"%s\",%.2f,%d,%.1f,%.1f,%d\n" % (d["kernel"], d["grid"], d["dur_us"],
                                                        d["dram_bytes"], d["tensor_pct"],
                                                        d["dram_pct"], d["regs"]))
    conv = [d for d in out if d["kernel"].startswith("conv_tc")]
    js = os.path.join(OUT, "ncu_summary.json")
    allj = json.load(open(js)) if os.path.exists(js) else {}
    allj["alexnet_bf16_b256"] = {
        "round": RND, "conv_launches": len(conv),
        "conv_dram_bytes_per_launch": int(statistics.mean(d["dram_bytes"] for d in conv)),
        "per_launch": conv, "fc": [d for d in out if d["kernel"].startswith("fc_tc")],
        "source": "ncu --set full --clock-control none (one capture of each kernel)"}
    json.dump(allj, open(js, "w"), indent=1)
    summary["ncu_full_alexnet_b256"] = out
other = os.path.join(RAW, "full_alexnet_b256_other_%s.ncu-rep" % RND)
if os.path.exists(other):
    # memory-bound kernels (LRN + pool, staging, pooling, softmax): DRAM bytes
    # and throughput, issue activity and occupancy
    raw = subprocess.run(["ncu", "-i", other, "--page", "raw", "--csv"], capture_output=True,
                         text=True).stdout.splitlines()
    rows = list(csv.reader(raw))
    h = rows[0]
    keys = ["Kernel Name", "Grid Size", "gpu__time_duration.sum", "dram__bytes_read.sum",
            "dram__bytes_write.sum", "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
            "sm__inst_issued.avg.pct_of_peak_sustained_active",
            "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread"]
    idx = [h.index(k) if k in h else -1 for k in keys]
    units = [rows[1][i] if i >= 0 else "" for i in idx]
    with open(os.path.join(OUT, "%s_ncu_full_alexnet_b256_other.csv" % RND), "w") as f:
        f.write("kernel,grid,dur_us,dram_bytes,dram_pct,issue_active_pct,warps_active_pct,regs\n")
        for r in rows[2:]:
            d = {k: (r[i] if i >= 0 else "0") for k, i in zip(keys, idx)}
            mb = lambda x: float(x) * (1e6 if "Mbyte" in units[3] else 1e9 if "Gbyte" in units[3] else 1e3)
            f.write("\"%s\",\"%s\",%.2f,%d,%.1f,%.1f,%.1f,%d\n" % (
                short(d["Kernel Name"]), d["Grid Size"], float(d["gpu__time_duration.sum"]),
                int(mb(d["dram__bytes_read.sum"]) + mb(d["dram__bytes_write.sum"])),
                float(d["gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed"]),
                float(d["sm__inst_issued.avg.pct_of_peak_sustained_active"]),
                float(d["sm__warps_active.avg.pct_of_peak_sustained_active"]),
                int(float(d["launch__registers_per_thread"]))))
print(json.dumps(summary, indent=1))
