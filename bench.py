#!/usr/bin/env python
"""bench.py -- headline benchmark of the B200-native P-CNN hot path.

Metric (BASELINE.json): images/sec of batched AlexNet / VGG-16 inference, with
the conv kernels' tensor-pipe fraction of the measured BF16 peak.

Default workload (N=1): BASELINE.json configs[1] -- AlexNet 227x227, exact
variants, BF16, batch 256 (top of the 1..256 sweep; the sweep itself is
reported under "sweep").  One step = one full pass of the hot path (staging,
5 conv + 2 LRN + 3 pool + 3 FC, softmax + entropy) over one batch.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]
                    [--net alexnet|vgg16] [--batch B] [--precision bf16|tf32|fp32]

N > 1 runs under torchrun (one process per GPU, NCCL): weights are broadcast
once from rank 0, every rank infers its own B images (weak scaling, images
regenerated per rank from their global index) and logits are all-gathered
every step.  The timed region is bracketed by barrier + synchronize, measured
with CUDA events on the launch stream, max over ranks.

--impl reference runs the FP64 CPU oracle (this tier's reference arm) on a
bounded sample per step; rank 0 only.
"""
import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import synth  # noqa: E402

METRIC = "images/sec AlexNet & VGG-16 vs batch (1/2/4/8 B200); conv tensor-pipe % of peak"
PAPER_CONTEXT = {
    "alexnet": "P:133 Table III: TitanX (Maxwell, FP32) batch 128: cuBLAS 131 ms (977 img/s), "
               "cuDNN 68 ms (1882 img/s), Nervana 31 ms (4129 img/s)",
    "vgg16": "P:139 Table III: TitanX batch 32: cuBLAS 165 ms (194 img/s), cuDNN 152 ms (211 img/s)",
}


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=50)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--net", default="alexnet", choices=["alexnet", "vgg16"])
    ap.add_argument("--batch", type=int, default=None)
    ap.add_argument("--global-batch", type=int, default=None,
                    help="strong scaling (configs[4]): split this many images over the ranks")
    ap.add_argument("--precision", default="bf16", choices=["bf16", "tf32", "fp32"])
    ap.add_argument("--no-sweep", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-seconds", type=float, default=12.0)
    a = ap.parse_args()
    if a.batch is None:
        a.batch = 256 if a.net == "alexnet" else 64
    a.warmup = max(a.warmup, 3)
    return a


# ------------------------------------------------------------------ clocks
class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled every 50 ms while the GPU
    is under the bench's load (warm-up, timed steps, graph replay, e2e); a
    timed region alone can be shorter than one sampling period."""
    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")
    NAMES = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]

    def __init__(self, n_gpus):
        self.n = n_gpus
        self.rows = []
        self.proc = None
        self.th = None
        self.active = False

    def start(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "--query-gpu=" + self.Q, "--format=csv,noheader,nounits",
                 "-lms", "50"], stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
        except OSError:
            self.proc = None
            return
        self.th = threading.Thread(target=self._read, daemon=True)
        self.th.start()

    def _read(self):
        for line in self.proc.stdout:
            parts = [p.strip() for p in line.split(",")]
            if len(parts) >= 9 and self.active:
                self.rows.append(parts)

    def mark(self, on):
        self.active = on

    def stop(self):
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except Exception:
                self.proc.kill()
        rows = [r for r in self.rows if r[0].isdigit() and int(r[0]) < max(self.n, 1)]
        if not rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": [], "samples": 0}
        sm = [float(r[1]) for r in rows if r[1].replace(".", "").isdigit()]
        smax = [float(r[2]) for r in rows if r[2].replace(".", "").isdigit()]
        pw = [float(r[3]) for r in rows if r[3].replace(".", "").isdigit()]
        reasons = sorted({n for r in rows for n, v in zip(self.NAMES, r[5:9]) if v == "Active"})
        return {"sm_mhz": statistics.median(sm) if sm else None,
                "sm_max_mhz": max(smax) if smax else None,
                "power_w_max": max(pw) if pw else None,
                "reasons": reasons, "samples": len(rows)}


# ------------------------------------------------------------------ helpers
def measured_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        return d, "measured (MEASURED_PEAKS.json)"
    return {"hbm_gbs": 6650.0, "bf16_tflops": 1590.0, "bf16_tflops_sustained": 1400.0}, \
        "fallback (B200_PROFILING.md)"


def ncu_traffic(net_name, precision, batch):
    """dram bytes per conv-kernel launch from the committed ncu --set full summary."""
    p = os.path.join(ROOT, "profiles", "ncu_summary.json")
    if not os.path.exists(p):
        return None
    try:
        with open(p) as f:
            d = json.load(f)
        key = "%s_%s_b%d" % (net_name, precision, batch)
        return d.get(key, {}).get("conv_dram_bytes_per_launch")
    except Exception:
        return None


def cpu_baseline(net, w, b, seconds):
    """The oracle as it stands, on a bounded sample of the same workload."""
    from oracle import oracle
    oracle.build()
    cores = os.cpu_count() or 1
    n_done, t0 = 0, time.perf_counter()
    chunk = max(1, min(cores, 8))
    while True:
        x = synth.images(n_done, chunk, net["in_shape"])
        oracle.run_net(net, w, b, x, threads=cores)
        n_done += chunk
        el = time.perf_counter() - t0
        if el >= seconds or n_done >= 512:
            break
    return {"value": n_done / el, "unit": "images/sec", "cores": cores, "kind": "oracle",
            "sample": "%d images of %s (FP64 direct loops, %d threads), %.1f s"
                      % (n_done, net["name"], cores, el)}


# ------------------------------------------------------------------ reference arm
def run_reference(a):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    from oracle import oracle
    oracle.build()
    net = synth.get_net(a.net)
    w, b = synth.net_params(net)
    cores = os.cpu_count() or 1
    per_step = 2 if a.net == "alexnet" else 1
    for i in range(a.warmup):
        oracle.run_net(net, w, b, synth.images(i * per_step, per_step, net["in_shape"]),
                       threads=cores)
    xs = [synth.images((a.warmup + i) * per_step, per_step, net["in_shape"])
          for i in range(a.steps)]
    t0 = time.perf_counter()
    for x in xs:
        oracle.run_net(net, w, b, x, threads=cores)
    el = time.perf_counter() - t0
    v = a.steps * per_step / el
    print(json.dumps({
        "impl": "reference", "metric": METRIC, "value": v, "unit": "images/sec",
        "n_gpus": a.gpus, "steps": a.steps, "warmup": a.warmup,
        "ms_per_step": el * 1000 / a.steps, "higher_is_better": True, "scaling": "weak",
        "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": {"workload": "%s_exact_b%d" % (a.net, a.batch), "net": a.net,
                   "batch": a.batch, "precision": "fp64 (oracle)"},
        "cpu_baseline": {"value": v, "unit": "images/sec", "cores": cores, "kind": "oracle",
                         "sample": "%d images per step (bounded sample of batch %d)"
                                   % (per_step, a.batch)},
        "e2e": {"value": v, "unit": "images/sec", "h2d_bytes_per_step": 0,
                "d2h_bytes_per_step": 0},
    }))


# ------------------------------------------------------------------ our arm
def main():
    a = parse()
    if a.impl == "reference":
        run_reference(a)
        return
    import torch
    import torch.distributed as dist

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local)
    if world > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    from paper_conf_hpca_songhcl17_b200 import pcnn
    from paper_conf_hpca_songhcl17_b200 import dist as pdist

    net = synth.get_net(a.net)
    B = a.batch
    if a.global_batch:                     # configs[4]: e.g. VGG-16 1024 images over N GPUs
        if a.global_batch % world:
            raise SystemExit("--global-batch must be a multiple of the GPU count")
        B = a.global_batch // world
    # weights: generated on rank 0, broadcast once over NCCL (C1)
    t_b = time.perf_counter()
    if world > 1:
        w, b, bcast_ms = pdist.broadcast_params(net, rank)
    else:
        w, b = synth.net_params(net)
        bcast_ms = 0.0
    n = pcnn.Net(net, w, b, max_batch=B, precision=a.precision, device=local)
    # inputs resident in HBM: this rank's images by global index (C2, no traffic)
    x_host = synth.images(rank * B, B, net["in_shape"])
    x = torch.from_numpy(x_host).cuda()
    out = torch.empty((B, n.out_elems), device="cuda")
    probs = torch.empty_like(out)
    ent = torch.empty((B,), device="cuda")
    gathered = torch.empty((world * B, n.out_elems), device="cuda") if world > 1 else None
    stream = torch.cuda.current_stream()

    def step():
        n.infer(x, out, probs, ent, stream=stream)
        if world > 1:
            dist.all_gather_into_tensor(gathered, out)        # C3: logits gather

    def barrier():
        if world > 1:
            dist.barrier()

    sampler = ClockSampler(world) if rank == 0 else None
    if sampler:
        sampler.start()
        time.sleep(0.3)
        sampler.mark(True)
    for _ in range(a.warmup):
        step()
    torch.cuda.synchronize()

    # ---------------- timed region (live per-layer events on the launch stream)
    n.set_layer_timing(True)
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    barrier()
    torch.cuda.synchronize()
    ev0.record(stream)
    for _ in range(a.steps):
        step()
    ev1.record(stream)
    torch.cuda.synchronize()
    barrier()
    n.set_layer_timing(False)
    ms = ev0.elapsed_time(ev1)
    layer_ms, nsteps = n.read_layer_timing()
    launches = n.last_launch_count()
    t = torch.tensor([ms], device="cuda")
    if world > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    ms_max = float(t.item())
    value = world * B * a.steps / (ms_max / 1000.0)

    # ---------------- same steps replayed from the captured CUDA graph
    for _ in range(2):
        step()
    barrier()
    torch.cuda.synchronize()
    ev0.record(stream)
    for _ in range(a.steps):
        step()
    ev1.record(stream)
    torch.cuda.synchronize()
    barrier()
    tg = torch.tensor([ev0.elapsed_time(ev1)], device="cuda")
    if world > 1:
        dist.all_reduce(tg, op=dist.ReduceOp.MAX)
    value_graph = world * B * a.steps / (float(tg.item()) / 1000.0)

    # ---------------- end to end through the host-buffer C-ABI call
    xh = torch.from_numpy(x_host).pin_memory()
    oh = torch.empty((B, n.out_elems)).pin_memory()
    ph = torch.empty((B, n.out_elems)).pin_memory()
    hh = torch.empty((B,)).pin_memory()
    for _ in range(2):
        n.infer_host(xh, oh, ph, hh, stream=stream)
    barrier()
    te0 = time.perf_counter()
    e2e_steps = max(3, min(a.steps, 20))
    for _ in range(e2e_steps):
        n.infer_host(xh, oh, ph, hh, stream=stream)
        if world > 1:
            dist.all_gather_into_tensor(gathered, out)
            torch.cuda.synchronize()
    te = torch.tensor([time.perf_counter() - te0], device="cuda")
    barrier()
    if world > 1:
        dist.all_reduce(te, op=dist.ReduceOp.MAX)
    e2e_value = world * B * e2e_steps / float(te.item())

    if sampler:
        sampler.mark(False)
    clocks = sampler.stop() if sampler else None

    # ---------------- board energy per image (NVML counter over >= 1 s of steps,
    # after the clock sampling of the timed / e2e regions;
    # the eq. 15 SoC denominator, DESIGN.md NEXT-4)
    from paper_conf_hpca_songhcl17_b200 import tuning as ptuning
    meter = ptuning.EnergyMeter(local)
    energy = None
    if meter.read_j() is not None:
        # the same step count on every rank (steps carry collectives): ~1 s
        # at the all-reduced step time
        n_e = max(10, int(1000.0 / max(ms_max / a.steps, 1e-3)))
        barrier()
        torch.cuda.synchronize()
        e0j, t0 = meter.read_j(), time.perf_counter()
        for _ in range(n_e):
            step()
        torch.cuda.synchronize()
        el = time.perf_counter() - t0
        dj = meter.read_j() - e0j
        energy = {"j_per_image": round(dj / (n_e * B), 6), "avg_power_w": round(dj / el, 1),
                  "window_s": round(el, 3), "source": "nvmlDeviceGetTotalEnergyConsumption "
                  "(board, this rank's GPU)"}


    # ---------------- per-layer plan, roofline of the dominant kernel (conv)
    infos = [n.query_layer(i, B) for i in range(n.n_layers)]
    conv_idx = [i for i, f in enumerate(infos) if f["kind"] == pcnn.CONV]
    conv_ms = sum(layer_ms[i] for i in conv_idx) / max(nsteps, 1)
    conv_flops = sum(infos[i]["flops"] for i in conv_idx)
    per_launch_flops = conv_flops / len(conv_idx)
    per_launch_s = conv_ms / 1000.0 / len(conv_idx)
    achieved = per_launch_flops / per_launch_s / 1e12
    peaks, peak_src = measured_peaks()
    # burst figure: the conv kernels run at the maximum SM clock inside the step
    # (power far below the cap; see "clocks"), and several layers measure above
    # the power-capped sustained figure, which is no ceiling for them
    if a.precision == "bf16":
        peak, peak_note = peaks["bf16_tflops"], "bf16 burst (cuBLAS 8192^3), " + peak_src
    elif a.precision == "tf32":
        peak, peak_note = peaks["bf16_tflops"] / 2, "tf32 = measured bf16 burst x 1/2 (nominal ratio), " + peak_src
    else:
        peak, peak_note = 2 * 148 * 128 * peaks.get("sm_max_mhz", 1965) * 1e6 / 1e12, \
            "FP32 FFMA: 2 x 148 SMs x 128 lanes x max SM clock (ALU peak)"
    total_step_ms = ms_max / a.steps
    per_layer = []
    for i, f in enumerate(infos):
        L = net["layers"][i]
        lm = layer_ms[i] / max(nsteps, 1)
        d = {"layer": L.get("name", str(i)), "ms": round(lm, 5)}
        if f["flops"] > 0:
            d["tflops"] = round(f["flops"] / (lm / 1000) / 1e12, 2) if lm > 0 else None
            d["tile"] = "%dx%d" % (f["tile_m"], f["tile_n"])
            d["grid"] = f["grid"]
            d["util_eq6"] = round(f["util"], 3)
            d["rec_eq9"] = round(f["rec"], 3)
        elif (f["kind"] in (pcnn.MAXPOOL, pcnn.AVGPOOL) and i > 0 and infos[i - 1]["kind"] == pcnn.LRN
              and os.environ.get("PCNN_NO_FUSE") != "1"):
            # LRN + pool run as ONE launch (runtime.cu run_lrn_pool): the pool's
            # event window is empty, so the pair's time and bytes (LRN input read
            # + pool output write = this pool layer's in + out bytes, since the
            # LRN output has the LRN input's shape) go on the LRN entry.
            d["fused_into"] = per_layer[-1]["layer"]
            pm = per_layer[-1]["ms"] + lm
            per_layer[-1]["gbs"] = round(f["bytes"] / (pm / 1000) / 1e9, 1) if pm > 0 else None
            per_layer[-1]["includes"] = d["layer"]
        else:
            d["gbs"] = round(f["bytes"] / (lm / 1000) / 1e9, 1) if lm > 0 else None
        per_layer.append(d)
    per_layer.append({"layer": "staging+softmax+unstage",
                      "ms": round(total_step_ms - sum(layer_ms) / max(nsteps, 1), 5)})

    res = {
        "metric": METRIC,
        "value": round(value, 1),
        "unit": "images/sec",
        "n_gpus": world,
        "steps": a.steps,
        "warmup": a.warmup,
        "ms_per_step": round(total_step_ms, 4),
        "higher_is_better": True,
        "scaling": "strong" if a.global_batch else "weak",
        "vs_baseline": None,
        "dtype": a.precision,
        "data": "synthetic (seeded He-normal weights, U[-128,128) images, BF16-representable)",
        "config": {"workload": "%s_exact_b%d" % (a.net, B), "net": a.net, "batch_per_gpu": B,
                   "global_batch": world * B, "precision": a.precision, "variants": "exact",
                   "parallelism": "dp%d" % world,
                   "l2": "inputs larger than L2: %d MB fp32 images per step + %d MB activations"
                         % (x.numel() * 4 // 2**20, B * 55 * 55 * 96 * 2 // 2**20)},
        "roofline": {"bound": "tensor", "kernel": "conv_tc_kernel (tcgen05 implicit GEMM)"
                     if a.precision != "fp32" else "conv_simt_kernel",
                     "achieved": round(achieved, 1), "peak": peak, "unit": "TFLOP/s",
                     "frac": round(achieved / peak, 4),
                     "traffic": ncu_traffic(a.net, a.precision, B),
                     "per_launch_flops": per_launch_flops,
                     "launches_per_step": len(conv_idx),
                     "conv_share_of_step": round(conv_ms / total_step_ms, 3),
                     "peak_source": peak_note,
                     "timing": "CUDA events recorded by libpcnn on the launch stream around "
                               "every layer of every timed step"},
        "e2e": {"value": round(e2e_value, 1), "unit": "images/sec",
                "h2d_bytes_per_step": int(x_host.nbytes),
                "d2h_bytes_per_step": int(oh.numel() * 4 + ph.numel() * 4 + hh.numel() * 4),
                "api": "pcnn_infer_host (pinned host buffers)"},
        "gpu_launches": int(launches * a.steps),
        "launches_per_step": launches,
        "value_graph_replay": round(value_graph, 1),
        "per_layer": per_layer,
        "weights_broadcast_ms": round(bcast_ms, 3),
        "energy": energy,
        "clocks": clocks,
        "paper_context": PAPER_CONTEXT[a.net],
    }

    # ---------------- batch sweep (configs[1]: batch 1..256) on rank 0, N=1
    if rank == 0 and world == 1 and not a.no_sweep:
        sweep = {}
        batches = [bb for bb in (1, 2, 4, 8, 16, 32, 64, 128, 256) if bb <= B]
        for bb in batches:
            xb = x[:bb]
            ob = out[:bb]
            pb = probs[:bb]
            hb = ent[:bb]
            for _ in range(3):
                n.infer(xb, ob, pb, hb, stream=stream)
            torch.cuda.synchronize()
            reps = max(5, min(200, 2000 // bb))
            ev0.record(stream)
            for _ in range(reps):
                n.infer(xb, ob, pb, hb, stream=stream)
            ev1.record(stream)
            torch.cuda.synchronize()
            t_ms = ev0.elapsed_time(ev1) / reps
            sweep[str(bb)] = {"ms": round(t_ms, 4), "img_s": round(bb / t_ms * 1000, 1)}
        res["sweep"] = sweep
        res["sweep_note"] = "graph replay, inputs resident; small batches fit in L2"

    if rank == 0 and world == 1 and not a.no_cpu_baseline:
        res["cpu_baseline"] = cpu_baseline(net, w, b, a.cpu_seconds)
    if rank == 0:
        print(json.dumps(res))
    n.close()
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
