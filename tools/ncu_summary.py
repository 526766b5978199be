"""Summarise an ncu report (raw page) into one line per kernel launch."""
import csv, subprocess, sys
rep = sys.argv[1]
out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(out.splitlines()))
hdr, units = rows[0], rows[1]
def g(r, name):
    try: return r[hdr.index(name)]
    except ValueError: return "-"
keys = [("dur_us", "gpu__time_duration.sum"), ("grid", "launch__grid_size"), ("block", "launch__block_size"),
        ("dramR_MB", "dram__bytes_read.sum"), ("dramW_MB", "dram__bytes_write.sum"),
        ("tensor%", "sm__ops_path_tensor_op_utchmma_src_bf16_dst_fp32_sparsity_off.avg.pct_of_peak_sustained_elapsed"),
        ("tensor_tf32%", "sm__ops_path_tensor_op_utchmma_src_tf32_dst_fp32_sparsity_off.avg.pct_of_peak_sustained_elapsed"),
        ("dram%", "dram__throughput.avg.pct_of_peak_sustained_elapsed"),
        ("l2%", "lts__throughput.avg.pct_of_peak_sustained_elapsed"),
        ("l1%", "l1tex__throughput.avg.pct_of_peak_sustained_active"),
        ("smem_wf", "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum"),
        ("regs", "launch__registers_per_thread")]
print("kernel," + ",".join(k for k, _ in keys))
for r in rows[2:]:
    print(g(r, "Kernel Name")[:28] + "," + ",".join(g(r, m) for _, m in keys))
