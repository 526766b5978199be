#!/usr/bin/env python
"""bench.py -- headline benchmark of the B200-native P-CNN hot path.

Metric (BASELINE.json): images/sec of batched AlexNet / VGG-16 inference, with
the conv kernels' tensor-pipe fraction of the measured BF16 peak.

Default workload (N=1): BASELINE.json configs[1] -- AlexNet 227x227, exact
variants, BF16, batch 256 (top of the 1..256 sweep).  One step = one full pass
of the hot path (staging, 5 conv + 2 LRN + 3 pool + 3 FC, softmax + entropy)
over one batch.  The same JSON line also carries (N=1, unless --no-extra):
  * "sweep": batch 1..256 with whole-pass ms, img/s and per-layer ms and
    roofline fractions (configs[1]);
  * "also": VGG-16 B=64 BF16 (configs[3], where the >= 60% conv target
    applies), VGG-16 B=64 TF32, AlexNet B=256 TF32, and VGG-16 with 1024
    images split over the ranks (configs[4]).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]
                    [--net alexnet|vgg16] [--batch B] [--precision bf16|tf32|fp32]

--gpus N > 1 runs one process per GPU over NCCL: launched by torchrun (the
driver does this), or, when started without torchrun, bench.py re-executes
itself under `torch.distributed.run --nproc-per-node N` (dist.relaunch).
Weights are broadcast once from rank 0; every rank infers its own B images
(weak scaling, images regenerated per rank from their global index) and the
logits are all-gathered every step.  The timed region is bracketed by
barrier + synchronize, measured with CUDA events on the launch stream, max
over ranks.

--impl reference runs the FP64 CPU oracle (this tier's reference arm) on a
bounded sample per step; rank 0 only.
"""
import argparse
import hashlib
import json
import os
import statistics
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
L2_BYTES = 126 * 2 ** 20


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
    ap.add_argument("--no-extra", action="store_true", help="skip the 'also' workloads")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--minimal", action="store_true",
                    help="profiling: only the warm-up and the timed steps of the main workload "
                         "(no graph-replay pass, e2e, energy, sweep or extras)")
    ap.add_argument("--cpu-seconds", type=float, default=12.0)
    ap.add_argument("--nccl", action="store_true",
                    help="run the NCCL data path (weight broadcast, logits all-gather) even on "
                         "one rank")
    a = ap.parse_args()
    if a.batch is None:
        a.batch = 256 if a.net == "alexnet" else 64
    a.warmup = max(a.warmup, 3)
    return a


# ------------------------------------------------------------------ clocks
class ClockSampler:
    """NVML clocks / power / throttle reasons of this rank's GPU, polled every
    ~2 ms from a thread while the bench runs; samples taken while `timed` is
    set are the timed region's (a 20-step AlexNet region lasts ~14 ms, far
    shorter than nvidia-smi's 50 ms period, hence NVML polling)."""
    REASONS = (("hw_slowdown", "nvmlClocksEventReasonHwSlowdown"),
               ("hw_thermal_slowdown", "nvmlClocksEventReasonHwThermalSlowdown"),
               ("sw_thermal_slowdown", "nvmlClocksEventReasonSwThermalSlowdown"),
               ("sw_power_cap", "nvmlClocksEventReasonSwPowerCap"),
               ("hw_power_brake", "nvmlClocksEventReasonHwPowerBrakeSlowdown"))

    def __init__(self, device):
        self.rows = []
        self.timed = False
        self.stop_ev = threading.Event()
        self.th = None
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(device)
            self.max_sm = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
        except Exception:
            self.nv = None

    def start(self):
        if self.nv is None:
            return
        self.th = threading.Thread(target=self._run, daemon=True)
        self.th.start()

    def _run(self):
        nv, h = self.nv, self.h
        while not self.stop_ev.is_set():
            try:
                sm = nv.nvmlDeviceGetClockInfo(h, nv.NVML_CLOCK_SM)
                pw = nv.nvmlDeviceGetPowerUsage(h) / 1000.0
                rs = nv.nvmlDeviceGetCurrentClocksEventReasons(h)
                self.rows.append((self.timed, sm, pw, rs))
            except Exception:
                pass
            time.sleep(0.002)

    def stop(self):
        self.stop_ev.set()
        if self.th:
            self.th.join(timeout=2)
        if self.nv is None or not self.rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": [], "samples": 0,
                    "source": "unavailable"}

        def summ(rows):
            if not rows:
                return None
            names = sorted({n for r in rows for n, attr in self.REASONS
                            if r[3] & getattr(self.nv, attr, 0)})
            return {"sm_mhz": statistics.median(r[1] for r in rows),
                    "sm_min_mhz": min(r[1] for r in rows),
                    "power_w_median": round(statistics.median(r[2] for r in rows), 1),
                    "power_w_max": round(max(r[2] for r in rows), 1),
                    "reasons": names, "samples": len(rows)}
        timed = summ([r for r in self.rows if r[0]])
        allr = summ(self.rows)
        out = dict(timed or allr)
        out["sm_max_mhz"] = self.max_sm
        out["scope"] = "timed region" if timed else "whole run (no sample inside the timed region)"
        out["whole_run"] = allr
        out["source"] = "NVML every ~2 ms (nvmlDeviceGetClockInfo / GetCurrentClocksEventReasons)"
        return out


# ------------------------------------------------------------------ helpers
def measured_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        return d, "measured (MEASURED_PEAKS.json)"
    return {"hbm_gbs": 6650.0, "bf16_tflops": 1590.0, "bf16_tflops_sustained": 1400.0}, \
        "fallback (B200_PROFILING.md)"


def tensor_peak(precision, peaks, peak_src):
    # burst figure: the timed steps are ms-long bursts (DESIGN.md §9b on
    # burst vs sustained); TF32 = BF16 x 1/2 (nominal ratio)
    if precision == "bf16":
        return peaks["bf16_tflops"], "bf16 burst (cuBLAS 8192^3), " + peak_src
    if precision == "tf32":
        return peaks["bf16_tflops"] / 2, "tf32 = measured bf16 burst x 1/2 (nominal ratio), " + peak_src
    return 2 * 148 * 128 * peaks.get("sm_max_mhz", 1965) * 1e6 / 1e12, \
        "FP32 FFMA: 2 x 148 SMs x 128 lanes x max SM clock (ALU peak)"


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
class Ctx:
    """Process-group state shared by the measurements."""

    def __init__(self, world, rank, local, dist_on=None):
        import torch
        import torch.distributed as dist
        self.torch, self.dist = torch, dist
        self.world, self.rank, self.local = world, rank, local
        self.dist_on = world > 1 if dist_on is None else dist_on   # NCCL group initialised
        self.stream = torch.cuda.current_stream()
        self.peaks, self.peak_src = measured_peaks()

    def barrier(self):
        if self.dist_on:
            self.dist.barrier()

    def max_over_ranks(self, v):
        t = self.torch.tensor([float(v)], device="cuda")
        if self.dist_on:
            self.dist.all_reduce(t, op=self.dist.ReduceOp.MAX)
        return float(t.item())


def layer_rooflines(n, net, infos, layer_ms, nsteps, precision, peaks, peak_src):
    """Per layer: ms, and the fraction of the layer's own roofline
    max(FLOPs / tensor peak, bytes / HBM) it reaches (conv / FC: both terms;
    LRN / pool: bytes).  An LRN + pool pair runs as one launch: its time and
    bytes (LRN input + pool output) go on the LRN entry."""
    from paper_conf_hpca_songhcl17_b200 import pcnn
    tpk, _ = tensor_peak(precision, peaks, peak_src)
    hbm = peaks["hbm_gbs"] * 1e9
    out = []
    for i, f in enumerate(infos):
        L = net["layers"][i]
        lm = layer_ms[i] / max(nsteps, 1)
        d = {"layer": L.get("name") or str(i), "ms": round(lm, 5)}
        if f["flops"] > 0:
            t_roof = max(f["flops"] / (tpk * 1e12), f["bytes"] / hbm)
            d["tflops"] = round(f["flops"] / (lm / 1000) / 1e12, 2) if lm > 0 else None
            d["bound"] = "tensor" if f["flops"] / (tpk * 1e12) >= f["bytes"] / hbm else "hbm"
            d["roofline_frac"] = round(t_roof / (lm / 1000), 3) if lm > 0 else None
            d["tile"] = "%dx%d" % (f["tile_m"], f["tile_n"])
            d["grid"] = f["grid"]
            d["util_eq6"] = round(f["util"], 3)
            d["rec_eq9"] = round(f["rec"], 3)
            if f["splits"] > 1:
                d["splits"] = f["splits"]
        elif (f["kind"] in (pcnn.MAXPOOL, pcnn.AVGPOOL) and i > 0 and infos[i - 1]["kind"] == pcnn.LRN
              and lm < 0.25 * out[-1]["ms"]):
            d["fused_into"] = out[-1]["layer"]
            pm = out[-1]["ms"] + lm
            out[-1]["gbs"] = round(f["bytes"] / (pm / 1000) / 1e9, 1) if pm > 0 else None
            out[-1]["roofline_frac"] = round(f["bytes"] / hbm / (pm / 1000), 3) if pm > 0 else None
            out[-1]["bound"] = "hbm"
            out[-1]["includes"] = d["layer"]
        else:
            d["gbs"] = round(f["bytes"] / (lm / 1000) / 1e9, 1) if lm > 0 else None
            d["bound"] = "hbm"
            d["roofline_frac"] = round(f["bytes"] / hbm / (lm / 1000), 3) if lm > 0 else None
        out.append(d)
    return out


def conv_roofline(n, infos, layer_ms, nsteps, precision, peaks, peak_src):
    from paper_conf_hpca_songhcl17_b200 import pcnn
    conv_idx = [i for i, f in enumerate(infos) if f["kind"] == pcnn.CONV]
    conv_ms = sum(layer_ms[i] for i in conv_idx) / max(nsteps, 1)
    conv_flops = sum(infos[i]["flops"] for i in conv_idx)
    per_launch_flops = conv_flops / len(conv_idx)
    per_launch_s = conv_ms / 1000.0 / len(conv_idx)
    achieved = per_launch_flops / per_launch_s / 1e12
    peak, note = tensor_peak(precision, peaks, peak_src)
    return {"bound": "tensor" if precision != "fp32" else "alu",
            "kernel": "conv_tc_kernel (tcgen05 implicit GEMM)" if precision != "fp32"
            else "conv_simt_kernel",
            "achieved": round(achieved, 1), "peak": round(peak, 1), "unit": "TFLOP/s",
            "frac": round(achieved / peak, 4), "per_launch_flops": per_launch_flops,
            "launches_per_step": len(conv_idx), "conv_ms_per_step": round(conv_ms, 5),
            "peak_source": note}


def timed_steps(ctx, step, steps, sampler=None):
    """EXACTLY `steps` calls of step() between barrier + synchronize, CUDA
    events on the launch stream; returns the max over ranks in ms."""
    torch = ctx.torch
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    ctx.barrier()
    torch.cuda.synchronize()
    if sampler:
        sampler.timed = True
    ev0.record(ctx.stream)
    for _ in range(steps):
        step()
    ev1.record(ctx.stream)
    torch.cuda.synchronize()
    if sampler:
        sampler.timed = False
    ctx.barrier()
    return ctx.max_over_ranks(ev0.elapsed_time(ev1))


def measure(ctx, net_name, precision, B, steps, warmup, sampler=None, e2e=False,
            global_batch=None, label=None, minimal=False):
    """One workload: build the net (weights broadcast once for N > 1), warm
    up, time `steps` steps with live per-layer events, then the same steps
    replayed from the cached CUDA graph; optionally the end-to-end host-buffer
    path.  Returns (result dict, net handle, params, inputs)."""
    torch = ctx.torch
    from paper_conf_hpca_songhcl17_b200 import dist as pdist
    from paper_conf_hpca_songhcl17_b200 import pcnn
    net = synth.get_net(net_name)
    world, rank = ctx.world, ctx.rank
    if global_batch:
        start, B = pdist.shard_range(global_batch, world, rank)
        if global_batch % world:
            raise SystemExit("--global-batch must be a multiple of the GPU count")
    else:
        start = rank * B
    if ctx.dist_on:
        w, b, bcast_ms = pdist.broadcast_params(net, rank)
    else:
        w, b = synth.net_params(net)
        bcast_ms = 0.0
    n = pcnn.Net(net, w, b, max_batch=B, precision=precision, device=ctx.local)
    x_host = synth.images(start, B, net["in_shape"])
    x = torch.from_numpy(x_host).cuda()
    out = torch.empty((B, n.out_elems), device="cuda")
    probs = torch.empty_like(out)
    ent = torch.empty((B,), device="cuda")
    gathered = torch.empty((world * B, n.out_elems), device="cuda") if ctx.dist_on else None

    def step():
        n.infer(x, out, probs, ent, stream=ctx.stream)
        if ctx.dist_on:
            ctx.dist.all_gather_into_tensor(gathered, out)        # C3: logits gather

    for _ in range(warmup):
        step()
    torch.cuda.synchronize()
    # (1) the headline: EXACTLY `steps` steps as the library runs them (each
    # pcnn_infer replays its captured CUDA graph; kernels overlap their
    # neighbours' launch and prologue through PDL)
    ms = timed_steps(ctx, step, steps, sampler)
    launches = n.last_launch_count()
    value = world * B * steps / (ms / 1000.0)
    # (2) the same steps with a CUDA event recorded on the launch stream after
    # every layer (no graph; the events serialise the launches): per-layer
    # durations for the rooflines
    n.set_layer_timing(True)
    ms_ev = timed_steps(ctx, step, steps)
    n.set_layer_timing(False)
    layer_ms, nsteps = n.read_layer_timing()
    torch.cuda.synchronize()
    logits = (gathered if ctx.dist_on else out).cpu().numpy()
    infos = [n.query_layer(i, B) for i in range(n.n_layers)]
    per_layer = layer_rooflines(n, net, infos, layer_ms, nsteps, precision, ctx.peaks,
                                ctx.peak_src)
    total_step_ms = ms / steps
    per_layer.append({"layer": "staging+softmax+unstage",
                      "ms": round(ms_ev / steps - sum(layer_ms) / max(nsteps, 1), 5)})
    act_bytes = sum(f["bytes"] for f in infos)
    res = {
        "workload": label or "%s_exact_b%d_%s" % (net_name, B, precision),
        "value": round(value, 1), "unit": "images/sec", "ms_per_step": round(total_step_ms, 4),
        "n_gpus": world, "batch_per_gpu": B, "global_batch": world * B, "precision": precision,
        "value_layer_events": round(world * B * steps / (ms_ev / 1000.0), 1),
        "timing": "value: graph replay of the timed steps; per_layer / roofline: a second "
                  "timed pass with per-layer CUDA events on the launch stream",
        "roofline": conv_roofline(n, infos, layer_ms, nsteps, precision, ctx.peaks, ctx.peak_src),
        "per_layer": per_layer, "gpu_launches": int(launches * steps),
        "launches_per_step": launches, "weights_broadcast_ms": round(bcast_ms, 3),
        "l2": "inputs + activations + weights per step = %.0f MB (%s L2's 126 MB)"
              % ((x_host.nbytes + act_bytes) / 2 ** 20,
                 "larger than" if x_host.nbytes + act_bytes > L2_BYTES else "within"),
        "logits_sha256": hashlib.sha256(np.ascontiguousarray(logits, np.float32).tobytes()).hexdigest(),
    }
    if e2e:
        # end to end through the host-buffer C-ABI calls (pinned host memory,
        # H2D of the images and D2H of logits / probs / entropy every step).
        # Headline: 8-bit pixels (the images' native format, pcnn_infer_host_u8,
        # network input = pixel - 128 on the device); also the fp32 form.
        oh = torch.empty((B, n.out_elems)).pin_memory()
        ph = torch.empty((B, n.out_elems)).pin_memory()
        hh = torch.empty((B,)).pin_memory()
        og = torch.empty((B, n.out_elems), device="cuda") if ctx.dist_on else None
        px_host = synth.pixels(start, B, net["in_shape"])
        forms = {
            "u8": (torch.from_numpy(px_host).pin_memory(),
                   "pcnn_infer_host_u8 (pinned uint8 pixels, mean 128 subtracted on the device)"),
            "f32": (torch.from_numpy(x_host).pin_memory(), "pcnn_infer_host (pinned fp32 images)"),
        }
        e2e_res = {}
        for form, (xh, api) in forms.items():
            def call():
                if form == "u8":
                    n.infer_host_u8(xh, oh, mean=[128.0] * net["in_shape"][0], probs=ph, entropy=hh,
                                    stream=ctx.stream)
                else:
                    n.infer_host(xh, oh, ph, hh, stream=ctx.stream)
            for _ in range(2):
                call()
            ctx.barrier()
            te0 = time.perf_counter()
            e2e_steps = max(3, min(steps, 20))
            for _ in range(e2e_steps):
                call()
                if ctx.dist_on:   # gather THIS step's logits (re-uploaded from the host result)
                    og.copy_(oh, non_blocking=True)
                    ctx.dist.all_gather_into_tensor(gathered, og)
                    torch.cuda.synchronize()
            te = time.perf_counter() - te0
            ctx.barrier()
            te = ctx.max_over_ranks(te)
            e2e_res[form] = {
                "value": round(world * B * e2e_steps / te, 1), "unit": "images/sec",
                "h2d_bytes_per_step": int(xh.numel() * xh.element_size() +
                                          (oh.numel() * 4 if ctx.dist_on else 0)),
                "d2h_bytes_per_step": int(oh.numel() * 4 + ph.numel() * 4 + hh.numel() * 4),
                "api": api + (" + all_gather of the step's logits" if ctx.dist_on else "")}
        res["e2e"] = dict(e2e_res["u8"])
        res["e2e"]["fp32_images"] = e2e_res["f32"]
    return res, n, (net, w, b), (x, out, probs, ent)


def batch_sweep(ctx, n, net, precision, bufs):
    """configs[1]: batch 1..B -- whole-pass ms (graph replay) and per-layer
    ms with roofline fractions (live events)."""
    torch = ctx.torch
    x, out, probs, ent = bufs
    B = x.shape[0]
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    sweep = {}
    for bb in [v for v in (1, 2, 4, 8, 16, 32, 64, 128, 256) if v <= B]:
        xb, ob, pb, hb = x[:bb], out[:bb], probs[:bb], ent[:bb]
        for _ in range(3):
            n.infer(xb, ob, pb, hb, stream=ctx.stream)
        torch.cuda.synchronize()
        reps = max(5, min(200, 2000 // bb))
        ev0.record(ctx.stream)
        for _ in range(reps):
            n.infer(xb, ob, pb, hb, stream=ctx.stream)
        ev1.record(ctx.stream)
        torch.cuda.synchronize()
        t_ms = ev0.elapsed_time(ev1) / reps
        n.set_layer_timing(True)
        for _ in range(5):
            n.infer(xb, ob, pb, hb, stream=ctx.stream)
        n.set_layer_timing(False)
        lms, ns = n.read_layer_timing()
        infos = [n.query_layer(i, bb) for i in range(n.n_layers)]
        pl = layer_rooflines(n, net, infos, lms, ns, precision, ctx.peaks, ctx.peak_src)
        cr = conv_roofline(n, infos, lms, ns, precision, ctx.peaks, ctx.peak_src)
        sweep[str(bb)] = {
            "ms": round(t_ms, 4), "img_s": round(bb / t_ms * 1000, 1),
            "conv_frac": cr["frac"],
            "layers": {d["layer"]: [d["ms"], d.get("roofline_frac")] for d in pl
                       if "fused_into" not in d}}
    return sweep


def main():
    a = parse()
    if a.impl == "reference":
        run_reference(a)
        return
    if a.gpus > 1 and "WORLD_SIZE" not in os.environ:
        # one process per GPU: re-execute under torchrun (rank 0 prints the line)
        from paper_conf_hpca_songhcl17_b200 import dist as pdist
        sys.exit(pdist.relaunch(a.gpus, [os.path.abspath(__file__)] + sys.argv[1:]))
    import torch
    import torch.distributed as dist

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local)
    use_dist = world > 1 or a.nccl
    if use_dist:
        if "MASTER_ADDR" not in os.environ:     # --nccl without torchrun: a 1-rank group
            os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=os.environ.get("MASTER_PORT", "29533"),
                              RANK="0", WORLD_SIZE="1", LOCAL_RANK="0")
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    from paper_conf_hpca_songhcl17_b200 import dist as pdist
    from paper_conf_hpca_songhcl17_b200 import tuning as ptuning
    pdist.check_world(a.gpus) if world > 1 else None
    if world == 1 and a.gpus != 1:
        raise SystemExit("--gpus %d but WORLD_SIZE=1" % a.gpus)
    ctx = Ctx(world, rank, local, dist_on=use_dist)

    sampler = ClockSampler(local)
    sampler.start()
    main_res, n, (net, w, b), bufs = measure(
        ctx, a.net, a.precision, a.batch, a.steps, a.warmup, sampler=sampler, e2e=not a.minimal,
        global_batch=a.global_batch, minimal=a.minimal)
    if a.minimal:
        sampler.stop()
        if rank == 0:
            print(json.dumps({"metric": METRIC, "value": main_res["value"], "unit": "images/sec",
                              "ms_per_step": main_res["ms_per_step"], "minimal": True,
                              "per_layer": main_res["per_layer"]}))
        n.close()
        if use_dist:
            dist.destroy_process_group()
        return
    B = main_res["batch_per_gpu"]

    # board energy per image (NVML counter over >= 1 s of steps; the eq. 15
    # SoC denominator, DESIGN.md NEXT-4)
    meter = ptuning.EnergyMeter(local)
    energy = None
    if meter.read_j() is not None:
        x, out, probs, ent = bufs
        n_e = max(10, int(1000.0 / max(main_res["ms_per_step"], 1e-3)))
        ctx.barrier()
        torch.cuda.synchronize()
        e0j, t0 = meter.read_j(), time.perf_counter()
        for _ in range(n_e):
            n.infer(x, out, probs, ent, stream=ctx.stream)
        torch.cuda.synchronize()
        el = time.perf_counter() - t0
        dj = meter.read_j() - e0j
        energy = {"j_per_image": round(dj / (n_e * B), 6), "avg_power_w": round(dj / el, 1),
                  "window_s": round(el, 3), "source": "nvmlDeviceGetTotalEnergyConsumption "
                  "(board, this rank's GPU)"}
    clocks = sampler.stop()

    res = {
        "metric": METRIC,
        "value": main_res["value"],
        "unit": "images/sec",
        "n_gpus": world,
        "gpus_active": world,
        "nccl": bool(use_dist),
        "steps": a.steps,
        "warmup": a.warmup,
        "ms_per_step": main_res["ms_per_step"],
        "higher_is_better": True,
        "scaling": "strong" if a.global_batch else "weak",
        "vs_baseline": None,
        "dtype": a.precision,
        "data": "synthetic (seeded He-normal weights, U[-128,128) images, BF16-representable)",
        "config": {"workload": main_res["workload"], "net": a.net, "batch_per_gpu": B,
                   "global_batch": world * B, "precision": a.precision, "variants": "exact",
                   "parallelism": "dp%d" % world, "l2": main_res["l2"]},
        "roofline": dict(main_res["roofline"], traffic=ncu_traffic(a.net, a.precision, B),
                         conv_share_of_step=round(main_res["roofline"]["conv_ms_per_step"]
                                                  / main_res["ms_per_step"], 3),
                         timing="conv time: CUDA events recorded by libpcnn on the launch "
                                "stream around every layer of a second timed pass of the same "
                                "steps"),
        "e2e": main_res["e2e"],
        "gpu_launches": main_res["gpu_launches"],
        "launches_per_step": main_res["launches_per_step"],
        "value_layer_events": main_res["value_layer_events"],
        "per_layer": main_res["per_layer"],
        "weights_broadcast_ms": main_res["weights_broadcast_ms"],
        "logits_sha256": main_res["logits_sha256"],
        "energy": energy,
        "clocks": clocks,
        "paper_context": PAPER_CONTEXT[a.net],
    }

    if rank == 0 and world == 1 and not a.no_sweep:
        res["sweep"] = batch_sweep(ctx, n, net, a.precision, bufs)
        res["sweep_note"] = ("ms: graph replay, inputs resident (small batches fit in L2); "
                             "layers: {name: [ms, fraction of the layer's roofline]}")
    n.close()

    if not a.no_extra:
        extra = []
        todo = [("vgg16", "bf16", 64, None), ("vgg16", "tf32", 64, None),
                ("alexnet", "tf32", 256, None)] if world == 1 else []
        todo.append(("vgg16", "bf16", None, 1024))           # configs[4]
        for (nn, pp, bb, gb) in todo:
            if (nn, pp, bb) == (a.net, a.precision, a.batch) and not gb:
                continue
            lab = ("vgg16_global1024_bf16 (configs[4], %d per GPU)" % (1024 // world)) if gb \
                else None
            r, nx, _, _ = measure(ctx, nn, pp, bb or 1, 10 if gb else 20, 3, global_batch=gb,
                                  label=lab)
            nx.close()
            r.pop("per_layer") if gb else None
            extra.append(r)
        res["also"] = extra

    if rank == 0 and world == 1 and not a.no_cpu_baseline:
        res["cpu_baseline"] = cpu_baseline(net, w, b, a.cpu_seconds)
    if rank == 0:
        print(json.dumps(res))
    if use_dist:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
